# r01j: GPU suite with batched k_reduce; A/B GALA_REDUCE_U=0 vs default; final bench lines + launch list + ncu
mkdir -p gpurun_out
make -s -j8 all >/dev/null 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/n_pytest_gpu.txt 2>&1; echo "exit $?" >> gpurun_out/n_pytest_gpu.txt
timeout 300 python __graft_entry__.py smoke > gpurun_out/n_smoke.txt 2>&1
AB='[{}]'
for C in lfr1m orkut; do echo "== reduce_u4 $C" >> gpurun_out/n_ab.txt; timeout 400 python tools/ab.py $C "$AB" >> gpurun_out/n_ab.txt 2>&1; done
make -s -B EXTRA=-DGALA_REDUCE_U=0 paper_conf_ppopp_wangllwm00z25_b200/libgala.so >/dev/null 2>&1
for C in lfr1m orkut; do echo "== reduce_u0 $C" >> gpurun_out/n_ab.txt; timeout 400 python tools/ab.py $C "$AB" >> gpurun_out/n_ab.txt 2>&1; done
make -s -B paper_conf_ppopp_wangllwm00z25_b200/libgala.so >/dev/null 2>&1
TAG=r01j
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/${TAG}_smi.txt
bash tools/profile_traffic.sh ${TAG} lfr1m:reduce,prune_bin,apply > gpurun_out/${TAG}_profile.log 2>&1
for C in lfr1m rmat_lj orkut; do
  timeout 600 python bench.py --config $C > gpurun_out/${TAG}_bench_$C.json 2> gpurun_out/${TAG}_bench_$C.err
done
timeout 600 python bench.py --impl reference --steps 2 --warmup 0 > gpurun_out/${TAG}_bench_reference_lfr1m.json 2>&1
timeout 900 python bench.py --config friendster_q > gpurun_out/${TAG}_bench_friendster_q.json 2> gpurun_out/${TAG}_bench_friendster_q.err
