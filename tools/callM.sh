# r01j: GPU suite with the pinned-buffer stash; e2e phase breakdown with teardown timing; bench lfr1m
mkdir -p gpurun_out
make -s -j8 all >/dev/null 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/m_pytest_gpu.txt 2>&1; echo "exit $?" >> gpurun_out/m_pytest_gpu.txt
GALA_DEBUG_FREE=1 timeout 300 python tools/e2e_breakdown.py lfr1m > gpurun_out/m_e2e_lfr1m.txt 2>&1
GALA_DEBUG_FREE=1 timeout 300 python tools/e2e_breakdown.py orkut > gpurun_out/m_e2e_orkut.txt 2>&1
timeout 600 python bench.py --config lfr1m > gpurun_out/m_bench_lfr1m.json 2> gpurun_out/m_bench_lfr1m.err
