#!/bin/bash
# A/B builds of libgbdtmo.so with compile-time knobs, for measurement only:
#   tools/ab_build.sh <name> "-DGBDTMO_HIST_SB=16 ..."   ->  build/ab/<name>/libgbdtmo.so
set -e
name=$1; flags=$2
out=build/ab/$name; mkdir -p $out
for f in paper_conf_icpp_liupw25_b200/csrc/*.cu; do
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Iinclude $flags \
       -c -o $out/$(basename $f .cu).o $f &
done
wait
nvcc -gencode arch=compute_100a,code=sm_100a -shared -o $out/libgbdtmo.so $out/*.o -lcudart
echo $out/libgbdtmo.so
