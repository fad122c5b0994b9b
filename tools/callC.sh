# pytest on the default build, bench rmat_lj, then block-kernel shape variants (A/B)
make -s -j8 all >/dev/null
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/c_pytest_gpu.txt 2>&1; echo "exit $?" >> gpurun_out/c_pytest_gpu.txt
timeout 600 python bench.py --config rmat_lj > gpurun_out/c_bench_rmat_lj.json 2> gpurun_out/c_bench_rmat_lj.err
timeout 300 python tools/level_profile.py rmat_lj '{"verbose":1}' > gpurun_out/c_verbose_rmat_lj.txt 2>&1
for V in "256 4" "512 4" "256 8" "512 2" "128 8"; do
  set -- $V
  make -s -B paper_conf_ppopp_wangllwm00z25_b200/libgala.so EXTRA="-DGALA_BLOCK_BT=$1 -DGALA_BLOCK_E=$2" > /dev/null 2>&1
  echo "== BT=$1 E=$2" >> gpurun_out/c_ab_block.txt
  timeout 300 python tools/ab.py orkut '[{}]' >> gpurun_out/c_ab_block.txt 2>&1
  timeout 300 python tools/ab.py rmat_lj '[{}]' >> gpurun_out/c_ab_block.txt 2>&1
done
make -s -B paper_conf_ppopp_wangllwm00z25_b200/libgala.so > /dev/null 2>&1
