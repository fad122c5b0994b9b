#!/bin/bash
# ncu pass: launch list of one gala_run (lfr1m), then one `ncu --set full` capture of every launch
# of the named kernel classes of one gala_run per config -> per-class DRAM traffic
# (profiles/traffic.json via tools/traffic_json.py) + metric summaries.  Reports go to /tmp
# (large); only the summaries land in gpurun_out/.
# usage: tools/profile_traffic.sh <tag> <config>:<class>[,<class>...] ...
#   e.g. tools/profile_traffic.sh r01e lfr1m:decide_warp,decide_small orkut:decide_block
set -x
TAG=$1; shift
mkdir -p gpurun_out /tmp/ncu
make -s >/dev/null
for LC in lfr1m orkut; do
  ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv \
      --log-file gpurun_out/${TAG}_launches_$LC.csv python tools/profile_run.py --config $LC > /dev/null 2>&1
  python tools/launches.py gpurun_out/${TAG}_launches_$LC.csv 40 > gpurun_out/${TAG}_launches_$LC.txt
done
declare -A RX=( [prune_bin]='k_prune_bin' [decide_single]='k_decide_single' [decide_small]='k_decide_small'
  [decide_warp]='k_decide_warp<[^,]*32, [^,]*128' [decide_warp512]='k_decide_warp<[^,]*32, [^,]*512' [decide_block]='k_decide_block'
  [decide_hub]='k_hub_|k_decide_cluster' [apply]='k_apply' [dp_update]='k_dp_|k_sm_flags' [reduce]='k_reduce'
  [phase2]='k_agg_|k_gather_flat|k_compact' )
for spec in "$@"; do
  C=${spec%%:*}; CL=${spec#*:}
  R=""
  for c in ${CL//,/ }; do R="${R:+$R|}${RX[$c]}"; done
  timeout 900 ncu --set full --clock-control none --import-source on --profile-from-start off \
      --kernel-name-base demangled -k "regex:^(void )?($R)" -o /tmp/ncu/${TAG}_$C -f \
      python tools/profile_run.py --config $C > gpurun_out/${TAG}_full_$C.log 2>&1
  python tools/traffic_json.py /tmp/ncu/${TAG}_$C.ncu-rep $C gpurun_out/${TAG}_traffic.json > /dev/null
  python tools/ncu_summary.py /tmp/ncu/${TAG}_$C.ncu-rep > gpurun_out/${TAG}_ncu_full_$C.txt
done
