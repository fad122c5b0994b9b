make -s -j8 all >/dev/null
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/e_pytest_gpu.txt 2>&1; echo "exit $?" >> gpurun_out/e_pytest_gpu.txt
timeout 300 python tools/ab.py lfr1m '[{}]' > gpurun_out/e_ab.txt 2>&1
timeout 300 python tools/ab.py orkut '[{}]' >> gpurun_out/e_ab.txt 2>&1
timeout 300 python tools/ab.py rmat_lj '[{}]' >> gpurun_out/e_ab.txt 2>&1
for V in "-DGALA_PRUNE_MINB=4" "-DGALA_W512_MINB=6" "-DGALA_PRUNE_MINB=4 -DGALA_W512_MINB=6"; do
  make -s -B paper_conf_ppopp_wangllwm00z25_b200/libgala.so EXTRA="$V" > /dev/null 2>&1
  echo "== $V" >> gpurun_out/e_ab.txt
  timeout 300 python tools/ab.py lfr1m '[{}]' >> gpurun_out/e_ab.txt 2>&1
  timeout 300 python tools/ab.py orkut '[{}]' >> gpurun_out/e_ab.txt 2>&1
done
make -s -B paper_conf_ppopp_wangllwm00z25_b200/libgala.so > /dev/null 2>&1
timeout 900 python bench.py --config friendster_q --steps 5 > gpurun_out/e_bench_friendster_q.json 2> gpurun_out/e_bench_friendster_q.err
timeout 1200 env GALA_XL=1 python -m pytest tests/test_gpu_parity.py -k friendster -x -q > gpurun_out/e_pytest_xl.txt 2>&1; echo "exit $?" >> gpurun_out/e_pytest_xl.txt
