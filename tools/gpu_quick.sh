#!/bin/bash
# Short GPU-box pass (no ncu): gpu tests, smoke, bench lines, per-level profile of one config.
# usage: tools/gpu_quick.sh <tag> [configs...]
TAG=${1:-q}; shift
CFGS=${@:-lfr1m rmat_lj orkut}
mkdir -p gpurun_out
make -s -j8 all >/dev/null
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/${TAG}_pytest_gpu.txt 2>&1
echo "pytest exit $?" >> gpurun_out/${TAG}_pytest_gpu.txt
timeout 300 python __graft_entry__.py smoke > gpurun_out/${TAG}_smoke.txt 2>&1
for C in $CFGS; do
  timeout 600 python bench.py --config $C > gpurun_out/${TAG}_bench_$C.json 2> gpurun_out/${TAG}_bench_$C.err
  timeout 300 python tools/level_profile.py $C > gpurun_out/${TAG}_levels_$C.txt 2>&1
done
