make -s -j8 all >/dev/null
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/g_pytest_gpu.txt 2>&1; echo "exit $?" >> gpurun_out/g_pytest_gpu.txt
AB='[{"block_split":0}, {}, {"block_split":1024}]'
for C in lfr1m orkut rmat_lj; do timeout 400 python tools/ab.py $C "$AB" >> gpurun_out/g_ab.txt 2>&1; done
timeout 900 python tools/ab.py friendster_q "$AB" >> gpurun_out/g_ab.txt 2>&1
