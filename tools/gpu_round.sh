#!/bin/bash
# One GPU-box pass: gpu tests (incl. full-size), bench lines for the three 1-GPU configs,
# launch list + ncu full captures (traffic per kernel class) on the headline config.
# usage: tools/gpu_round.sh <tag> [skip_tests]
TAG=${1:-r01e}
mkdir -p gpurun_out
make -s -j8 all >/dev/null
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/${TAG}_smi.txt
if [ -z "$2" ]; then
  timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/${TAG}_pytest_gpu.txt 2>&1
  echo "pytest exit $?" >> gpurun_out/${TAG}_pytest_gpu.txt
  timeout 600 python __graft_entry__.py smoke > gpurun_out/${TAG}_smoke.txt 2>&1
fi
bash tools/profile_traffic.sh ${TAG} > gpurun_out/${TAG}_profile.log 2>&1
for C in lfr1m rmat_lj orkut; do
  timeout 600 python bench.py --config $C > gpurun_out/${TAG}_bench_$C.json 2> gpurun_out/${TAG}_bench_$C.err
done
timeout 600 python bench.py --impl reference --steps 2 --warmup 0 > gpurun_out/${TAG}_bench_reference.json 2>&1
