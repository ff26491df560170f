#!/bin/bash
# Round evidence on one B200 (run under gpurun from the repo root):
#   1. the default bench line                    -> gpurun_out/prof/bench_suite.json
#   2. the ncu launch list of a short bench run   -> gpurun_out/prof/launches.csv
#   3. --set full captures of each suite kernel under none / intra_reg /
#      intra_smem / inter_group                   -> gpurun_out/prof/full/*.ncu-rep
# Summarise here with tools/ncu_summary.py and tools/launch_summary.py.
set -u
out=gpurun_out/prof
mkdir -p $out/full
timeout 600 python bench.py > $out/bench.log 2>&1; grep '^{' $out/bench.log | tail -1 > $out/bench_suite.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $out/launches.csv \
  python bench.py --steps 2 --warmup 1 --no-cpu-baseline --e2e-steps 0 --energy-seconds 0 --extra-variants "" \
  > $out/launches_bench.log 2>&1
for kv in "binarysearch bins_kernel" "fwt fwt_kernel" "prefixsum ps_scan_kernel" "reduction red_partial_kernel" \
          "transpose tr_kernel" "sobel sobel_kernel"; do
  set -- $kv
  for vv in "none 0" "intra_smem 1" "intra_reg 2" "inter_group 3"; do
    set -- $kv $vv
    timeout 200 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
      -k "regex:$2<.int.$4, .int.0" -s 1 -c 1 -o $out/full/$1_$3 \
      python tools/prof_run.py suite $1 $3 2 > $out/full/$1_$3.log 2>&1
  done
done
ls -la $out $out/full
