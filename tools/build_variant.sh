#!/bin/bash
# Build libgala.so with extra compile-time flags into scratch/variants/<name>/ (a package copy), for
# A/B runs of compile-time choices: PYTHONPATH=scratch/variants/<name>:. python tools/ab.py ...
# usage: tools/build_variant.sh <name> "<nvcc -D flags>"
set -e
ROOT=$(cd "$(dirname "$0")/.." && pwd)
PKG=paper_conf_ppopp_wangllwm00z25_b200
OUT=$ROOT/scratch/variants/$1/$PKG
mkdir -p "$OUT"
cp "$ROOT/$PKG/__init__.py" "$OUT/"
/usr/local/cuda/bin/nvcc $2 -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -lineinfo -Xcompiler -fPIC,-O3 \
    -I"$ROOT/include" --expt-relaxed-constexpr -shared -o "$OUT/libgala.so" "$ROOT"/$PKG/csrc/*.cu -ldl
echo "built $OUT/libgala.so ($2)"
