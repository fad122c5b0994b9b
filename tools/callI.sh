make -s -j8 all >/dev/null
timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "graph_mode" > gpurun_out/i_pytest_graph.txt 2>&1; echo "exit $?" >> gpurun_out/i_pytest_graph.txt
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/i_pytest_gpu.txt 2>&1; echo "exit $?" >> gpurun_out/i_pytest_gpu.txt
AB='[{}, {"agg_bound":0}]'
for C in lfr1m orkut rmat_lj; do timeout 400 python tools/ab.py $C "$AB" >> gpurun_out/i_ab.txt 2>&1; done
timeout 900 python tools/ab.py friendster_q "$AB" >> gpurun_out/i_ab.txt 2>&1
