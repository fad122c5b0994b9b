#!/bin/bash
# Launch list (lfr1m) + one `ncu --set full` capture of every phase-1 kernel of one gala_run per
# config, reduced to profiles-ready summaries and per-class DRAM traffic (profiles/traffic.json).
# usage: tools/profile_traffic.sh <tag>
set -x
TAG=${1:-r01e}
mkdir -p gpurun_out
make -s >/dev/null
ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv \
    --log-file gpurun_out/${TAG}_launches_lfr1m.csv python tools/profile_run.py --config lfr1m > /dev/null 2>&1
K='regex:^k_(prune_bin|decide|hub_|apply|dp_|reduce|sm_flags)'
for C in lfr1m orkut rmat_lj; do
  timeout 1200 ncu --set full --clock-control none --import-source on --profile-from-start off -k "$K" \
      -o gpurun_out/${TAG}_full_$C -f python tools/profile_run.py --config $C > gpurun_out/${TAG}_full_$C.log 2>&1
  python tools/traffic_json.py gpurun_out/${TAG}_full_$C.ncu-rep $C gpurun_out/${TAG}_traffic.json > /dev/null
  python tools/ncu_summary.py gpurun_out/${TAG}_full_$C.ncu-rep > gpurun_out/${TAG}_ncu_full_$C.txt
  rm -f gpurun_out/${TAG}_full_$C.ncu-rep   # large; the summaries and traffic.json are kept
done
cp gpurun_out/${TAG}_traffic.json profiles/traffic.json
