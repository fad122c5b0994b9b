# r01j: GPU suite with the parallel reduce tail; A/B GALA_REDUCE_PTAIL=0; bench lfr1m
mkdir -p gpurun_out
L=paper_conf_ppopp_wangllwm00z25_b200/libgala.so
make -s -j8 all >/dev/null 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/r_pytest_gpu.txt 2>&1; echo "exit $?" >> gpurun_out/r_pytest_gpu.txt
timeout 300 python __graft_entry__.py smoke > gpurun_out/r_smoke.txt 2>&1
AB='[{}]'
for C in lfr1m orkut; do echo "== ptail1 $C" >> gpurun_out/r_ab.txt; timeout 400 python tools/ab.py $C "$AB" >> gpurun_out/r_ab.txt 2>&1; done
make -s -B EXTRA=-DGALA_REDUCE_PTAIL=0 $L >/dev/null 2>&1
for C in lfr1m orkut; do echo "== ptail0 $C" >> gpurun_out/r_ab.txt; timeout 400 python tools/ab.py $C "$AB" >> gpurun_out/r_ab.txt 2>&1; done
make -s -B $L >/dev/null 2>&1
timeout 600 python bench.py --config lfr1m > gpurun_out/r_bench_lfr1m.json 2> gpurun_out/r_bench_lfr1m.err
