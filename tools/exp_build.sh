#!/bin/bash
# Experiment builds: tools/exp_build.sh NAME "k_a.cu k_b.cu" "-DFOO=1 ..." -> build_exp/NAME.so
# (a source given as a path, e.g. build_exp/src/k_sobel.cu, replaces csrc's TU of
# the same name)
# (librmt.so with the listed translation units recompiled under extra defines;
# select it with RMT_LIB=build_exp/NAME.so).  Not part of the product build.
set -e
name=$1; srcs=$2; defs=$3
root=$(cd "$(dirname "$0")/.." && pwd)
pkg=$root/paper_conf_isca_waddenlgss14_b200
mkdir -p $root/build_exp
objs=$(ls $pkg/build/*.o)
pids=()
for src in $srcs; do
  base=$(basename $src .cu)
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -fmad=false -Xcompiler -fPIC,-O2 \
    --expt-relaxed-constexpr -I $root/include -I $pkg/csrc $defs -c $(case $src in */*) echo $src;; *) echo $pkg/csrc/$base.cu;; esac) \
    -o $root/build_exp/$name.$base.o &
  pids+=($!)
  objs=$(echo "$objs" | grep -v "/$base.o$")
  objs=$(printf "%s\n%s" "$objs" "$root/build_exp/$name.$base.o")
done
for p in "${pids[@]}"; do wait $p; done
nvcc -gencode arch=compute_100a,code=sm_100a -shared -cudart static -o $root/build_exp/$name.so $objs
echo $root/build_exp/$name.so
