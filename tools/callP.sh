# r01j: prune_bin eager loads A/B: EAGER=1 MINB=4 (default build), EAGER=1 MINB=3, EAGER=0 MINB=4 (previous)
mkdir -p gpurun_out
L=paper_conf_ppopp_wangllwm00z25_b200/libgala.so
make -s -j8 all >/dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "prune or graph_mode or weighted" > gpurun_out/p_pytest.txt 2>&1; echo "exit $?" >> gpurun_out/p_pytest.txt
AB='[{}]'
for V in "eager_minb4:" "eager_minb3:-DGALA_PRUNE_MINB=3" "lazy_minb4:-DGALA_PRUNE_EAGER=0"; do
  N=${V%%:*}; F=${V#*:}
  make -s -B EXTRA="$F" $L >/dev/null 2>&1
  for C in lfr1m orkut rmat_lj; do echo "== $N $C" >> gpurun_out/p_ab.txt; timeout 400 python tools/ab.py $C "$AB" >> gpurun_out/p_ab.txt 2>&1; done
done
make -s -B $L >/dev/null 2>&1
