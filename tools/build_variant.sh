#!/bin/bash
# Build an experimental libnestgpu variant with extra nvcc defines into $1.
# usage: tools/build_variant.sh out.so -DNG_B_RPT=16 -DNG_B_STAGES=3
set -e
OUT=$1; shift
D=$(mktemp -d)
ROOT=$(cd "$(dirname "$0")/.." && pwd)
CS=$ROOT/paper_conf_icde_floratosxwgylz21_b200/csrc
for f in $CS/*.cu $CS/*.cpp; do
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-O3 --expt-relaxed-constexpr \
    -I$ROOT/include -I$CS "$@" -x cu -c $f -o $D/$(basename $f).o &
done
wait
nvcc -gencode arch=compute_100a,code=sm_100a -shared -cudart static -o $OUT $D/*.o
rm -rf $D
