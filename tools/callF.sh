make -s -j8 all >/dev/null
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/f_pytest_gpu.txt 2>&1; echo "exit $?" >> gpurun_out/f_pytest_gpu.txt
AB='[{}, {"agg_big_ent":16384}, {"agg_big_ent":4096}]'
for C in lfr1m orkut rmat_lj; do timeout 400 python tools/ab.py $C "$AB" >> gpurun_out/f_ab.txt 2>&1; done
timeout 900 python tools/ab.py friendster_q "$AB" >> gpurun_out/f_ab.txt 2>&1
make -s -B paper_conf_ppopp_wangllwm00z25_b200/libgala.so EXTRA="-DGALA_WARP_PREFETCH=0" > /dev/null 2>&1
echo "== no prefetch" >> gpurun_out/f_ab.txt
for C in lfr1m orkut rmat_lj; do timeout 400 python tools/ab.py $C '[{}]' >> gpurun_out/f_ab.txt 2>&1; done
make -s -B paper_conf_ppopp_wangllwm00z25_b200/libgala.so > /dev/null 2>&1
timeout 600 python tools/level_profile.py friendster_q '{"verbose":1}' > gpurun_out/f_verbose_friendster_q.txt 2>&1
