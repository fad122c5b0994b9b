# r01j: GPU suite after the creation-path change; e2e phase breakdown; step-time outliers vs clock sampler
mkdir -p gpurun_out
make -s -j8 all >/dev/null 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/l_pytest_gpu.txt 2>&1; echo "exit $?" >> gpurun_out/l_pytest_gpu.txt
timeout 300 python tools/e2e_breakdown.py lfr1m > gpurun_out/l_e2e_lfr1m.txt 2>&1
timeout 300 python tools/e2e_breakdown.py orkut > gpurun_out/l_e2e_orkut.txt 2>&1
timeout 600 python tools/step_times.py orkut > gpurun_out/l_steps_orkut.txt 2>&1
timeout 600 python bench.py --config lfr1m > gpurun_out/l_bench_lfr1m.json 2> gpurun_out/l_bench_lfr1m.err
