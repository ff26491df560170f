#!/bin/bash
# usage: tools/ncu_suite.sh OUTDIR CONFIG "kernel:variant:regex:count ..."
# regex matches the demangled kernel name, e.g. 'tr_kernel<2, 0>'
out=$1; cfg=$2; shift 2
mkdir -p $out
for spec in "$@"; do
  IFS=: read k v rx c <<< "$spec"
  ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
      -k "regex:$rx" -s $c -c $c -o $out/${k}_${v} \
      python tools/prof_run.py $cfg $k $v 2 > $out/${k}_${v}.log 2>&1
done
