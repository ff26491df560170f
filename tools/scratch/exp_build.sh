#!/bin/bash
# Experiment builds: tools/exp_build.sh NAME SRC.cu "-DFOO=1 ..." -> build_exp/NAME.so
# (librmt.so with one translation unit recompiled under extra defines; select
# it with RMT_LIB=build_exp/NAME.so).  Not part of the product build.
set -e
name=$1; src=$2; defs=$3
root=$(cd "$(dirname "$0")/.." && pwd)
pkg=$root/paper_conf_isca_waddenlgss14_b200
mkdir -p $root/build_exp
base=$(basename $src .cu)
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -fmad=false -Xcompiler -fPIC,-O2 \
  --expt-relaxed-constexpr -I $root/include $defs -c $pkg/csrc/$base.cu -o $root/build_exp/$name.$base.o
objs=$(ls $pkg/build/*.o | grep -v "/$base.o$")
nvcc -gencode arch=compute_100a,code=sm_100a -shared -cudart static -o $root/build_exp/$name.so $objs $root/build_exp/$name.$base.o
echo $root/build_exp/$name.so
