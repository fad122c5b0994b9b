# r01i: full GPU suite after the smem-attribute fix, then early-exit A/B (build variants)
mkdir -p gpurun_out
make -s -j8 all >/dev/null 2>&1
timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "graph_mode or across_handles" > gpurun_out/j_pytest_graph.txt 2>&1; echo "exit $?" >> gpurun_out/j_pytest_graph.txt
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/j_pytest_gpu.txt 2>&1; echo "exit $?" >> gpurun_out/j_pytest_gpu.txt
timeout 300 python __graft_entry__.py smoke > gpurun_out/j_smoke.txt 2>&1
AB='[{}]'
for C in lfr1m orkut rmat_lj; do echo "== new $C" >> gpurun_out/j_ab.txt; timeout 400 python tools/ab.py $C "$AB" >> gpurun_out/j_ab.txt 2>&1; done
make -s -B EXTRA=-DGALA_EARLY_EXIT=0 paper_conf_ppopp_wangllwm00z25_b200/libgala.so >/dev/null 2>&1
for C in lfr1m orkut rmat_lj; do echo "== noexit $C" >> gpurun_out/j_ab.txt; timeout 400 python tools/ab.py $C "$AB" >> gpurun_out/j_ab.txt 2>&1; done
make -s -B paper_conf_ppopp_wangllwm00z25_b200/libgala.so >/dev/null 2>&1
