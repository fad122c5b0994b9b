# r01i: full GPU suite at HEAD; rmat/orkut A/B of the r01h build (scratch/ab_old) vs HEAD
mkdir -p gpurun_out
make -s -j8 all >/dev/null 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/k_pytest_gpu.txt 2>&1; echo "exit $?" >> gpurun_out/k_pytest_gpu.txt
AB='[{}]'
for C in rmat_lj lfr1m; do
  echo "== head $C" >> gpurun_out/k_ab.txt; timeout 400 python tools/ab.py $C "$AB" >> gpurun_out/k_ab.txt 2>&1
  echo "== r01h $C" >> gpurun_out/k_ab.txt; GALA_LIB_PATH=scratch/ab_old/libgala.so timeout 400 python tools/ab.py $C "$AB" >> gpurun_out/k_ab.txt 2>&1
done
TAG=r01i
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/${TAG}_smi.txt
bash tools/profile_traffic.sh ${TAG} lfr1m:decide_warp,decide_small,prune_bin,reduce,dp_update > gpurun_out/${TAG}_profile.log 2>&1
for C in lfr1m rmat_lj orkut; do
  timeout 600 python bench.py --config $C > gpurun_out/${TAG}_bench_$C.json 2> gpurun_out/${TAG}_bench_$C.err
done
timeout 600 python bench.py --impl reference --steps 2 --warmup 0 > gpurun_out/${TAG}_bench_reference_lfr1m.json 2>&1
timeout 900 python bench.py --config friendster_q > gpurun_out/${TAG}_bench_friendster_q.json 2> gpurun_out/${TAG}_bench_friendster_q.err
