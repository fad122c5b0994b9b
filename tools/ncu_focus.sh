#!/bin/bash
# Focused ncu --set full capture (with source) of selected launches of one config's run.
# usage: tools/ncu_focus.sh <tag> <config> <kernel-regex> <launch-count> [launch-skip]
# Writes gpurun_out/<tag>_<config>.ncu-rep plus a metric summary and per-kernel top source lines.
TAG=$1; C=$2; RX=$3; CNT=$4; SKIP=${5:-0}
mkdir -p gpurun_out
make -s >/dev/null
timeout 1500 ncu --set full --clock-control none --import-source on --profile-from-start off \
    --kernel-name-base demangled -k "regex:$RX" --launch-skip $SKIP --launch-count $CNT \
    -o gpurun_out/${TAG}_$C -f python tools/profile_run.py --config $C > gpurun_out/${TAG}_$C.log 2>&1
python tools/ncu_summary.py gpurun_out/${TAG}_$C.ncu-rep > gpurun_out/${TAG}_summary_$C.txt 2>&1
