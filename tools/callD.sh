make -s -j8 all >/dev/null
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/d_pytest_gpu.txt 2>&1; echo "exit $?" >> gpurun_out/d_pytest_gpu.txt
for C in lfr1m rmat_lj orkut; do
  timeout 600 python bench.py --config $C > gpurun_out/d_bench_$C.json 2> gpurun_out/d_bench_$C.err
done
timeout 1200 bash tools/profile_traffic.sh d lfr1m:decide_warp,decide_small,decide_warp512,prune_bin,dp_update,reduce,apply,decide_block,decide_single orkut:decide_block > gpurun_out/d_profile.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on --profile-from-start off --kernel-name-base demangled \
   -k 'regex:k_decide_warp<[^,]*32, [^,]*128' -s 2 -c 1 -o gpurun_out/d_src_warp128 -f python tools/profile_run.py --config lfr1m > gpurun_out/d_src.log 2>&1
