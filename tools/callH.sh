# round measurement: gpu tests, smoke, bench lines (4 configs), reference arm, ncu traffic/launches
TAG=${1:-r01h}
make -s -j8 all >/dev/null
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/${TAG}_smi.txt
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/${TAG}_pytest_gpu.txt 2>&1; echo "exit $?" >> gpurun_out/${TAG}_pytest_gpu.txt
timeout 300 python __graft_entry__.py smoke > gpurun_out/${TAG}_smoke.txt 2>&1
for C in lfr1m rmat_lj orkut; do
  timeout 600 python bench.py --config $C > gpurun_out/${TAG}_bench_$C.json 2> gpurun_out/${TAG}_bench_$C.err
done
timeout 900 python bench.py --config friendster_q --steps 5 > gpurun_out/${TAG}_bench_friendster_q.json 2> gpurun_out/${TAG}_bench_friendster_q.err
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/${TAG}_bench_reference.json 2>&1
timeout 1500 bash tools/profile_traffic.sh ${TAG} lfr1m:decide_warp,decide_small,decide_warp512,prune_bin,dp_update,reduce,apply,decide_block,decide_single orkut:decide_block rmat_lj:decide_block > gpurun_out/${TAG}_profile.log 2>&1
