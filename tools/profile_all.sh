#!/bin/bash
# GPU-box profiling pass: bench line, ncu launch list, full captures of the top kernels.
# usage: tools/profile_all.sh <tag> [config]
set -x
TAG=${1:-r01}; CFG=${2:-lfr1m}
mkdir -p gpurun_out
make -s >/dev/null
python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv \
    --log-file gpurun_out/${TAG}_launches.csv python tools/profile_run.py --config $CFG > /dev/null 2>&1
for K in k_decide_warp k_decide_small k_dp_full k_dp_delta k_prune_bin; do
  ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:$K -s 2 -c 2 \
      -o gpurun_out/${TAG}_full_$K -f python tools/profile_run.py --config $CFG > /dev/null 2>&1
done
