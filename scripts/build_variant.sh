#!/bin/bash
# Experiments only: build libgsh.so with extra nvcc defines into build/var_<name>/libgsh.so.
# Usage: build_variant.sh NAME "-DFOO=1 -DBAR=2"
set -e
NAME=$1; DEFS=$2
OUT=build/var_$NAME
mkdir -p $OUT
for f in paper_conf_icde_caic24_b200/csrc/*.cu; do
  /usr/local/cuda/bin/nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -lineinfo -Xcompiler -fPIC \
    -Xcompiler -fvisibility=hidden -Iinclude $DEFS -c $f -o $OUT/$(basename $f .cu).o &
done
wait
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -shared -cudart static -o $OUT/libgsh.so $OUT/*.o
echo built $OUT/libgsh.so
