# r01j: decide_small shape A/B (vertices in flight per 16/32-lane group, blocks per SM)
mkdir -p gpurun_out
L=paper_conf_ppopp_wangllwm00z25_b200/libgala.so
make -s -j8 all >/dev/null 2>&1
AB='[{}]'
for V in "default:" "u32_2:-DGALA_U32=2" "u16_2:-DGALA_U16=2" "minb3:-DGALA_SMALL_MINB=3"; do
  N=${V%%:*}; F=${V#*:}
  make -s -B EXTRA="$F" $L >/dev/null 2>&1
  for C in lfr1m orkut rmat_lj; do echo "== $N $C" >> gpurun_out/q_ab.txt; timeout 400 python tools/ab.py $C "$AB" >> gpurun_out/q_ab.txt 2>&1; done
done
make -s -B $L >/dev/null 2>&1
