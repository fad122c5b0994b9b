make -s -j8 all >/dev/null
timeout 300 python tools/level_profile.py rmat_lj '{"verbose":1}' > gpurun_out/r01e_verbose_rmat_lj.txt 2>&1
timeout 400 python tools/ab.py orkut '[{}, {"hub_smem_slots":4096}, {"hub_smem_slots":2048}, {"hub_smem_slots":16384}]' > gpurun_out/r01e_ab_orkut_smem.txt 2>&1
timeout 1200 bash tools/profile_traffic.sh r01e lfr1m:decide_warp orkut:decide_block rmat_lj:decide_block,phase2 > gpurun_out/r01e_profile.log 2>&1
