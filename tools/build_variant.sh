#!/bin/bash
# Build libmoment.so with extra nvcc defines into another path, for A/B runs (tools/ab_lib.sh, MOMENT_LIB_PATH).
# usage: tools/build_variant.sh OUT.so "-DNAME=V ..."
OUT=$1; DEFS=$2; T=$(mktemp -d)
for s in paper_conf_sc_shi0s0x0w25_b200/csrc/*.cu paper_conf_sc_shi0s0x0w25_b200/csrc/*.cpp; do
  x=""; [[ $s == *.cpp ]] && x="-x cu"
  /usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -Xcompiler -fPIC -lineinfo \
    --expt-relaxed-constexpr -I include -I paper_conf_sc_shi0s0x0w25_b200/csrc $DEFS $x -c $s -o $T/$(basename $s).o &
done; wait
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -shared -o $OUT $T/*.o -cudart static && rm -rf $T
