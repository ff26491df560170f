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
# cfg kernel capture-name kernel-regex skip
for kv in "suite binarysearch binarysearch bins_kernel 1" "suite fwt fwt_p1 fwt_p1_kernel 1" "suite fwt fwt_ps fwt_ps_kernel 1" \
          "suite prefixsum prefixsum ps_scan_kernel 1" "suite reduction reduction red_partial_kernel 1" \
          "suite transpose transpose tr_kernel 1" "suite sobel sobel sobel_kernel 1" \
          "fwdct dct dct dct_kernel 1" "fwdct floydwarshall fw_pass fw_pass_kernel 300"; do
  set -- $kv
  for vv in "none 0" "intra_smem 1" "intra_reg 2" "inter_group 3"; do
    set -- $kv $vv
    reps=2; [ "$2" = floydwarshall ] && reps=1
    timeout 300 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
      -k "regex:$4<.int.$7, .int.0" -s $5 -c 1 -o $out/full/$3_$6 \
      python tools/prof_run.py $1 $2 $6 $reps > $out/full/$3_$6.log 2>&1
  done
done
ls -la $out $out/full
# summarise on the box (the .ncu-rep files together exceed gpurun's 64 MiB
# copy-back limit); keep the dominant kernel's report only
python tools/ncu_summary.py $out/full/*.ncu-rep --json $out/ncu_full_summary.json > $out/ncu_full_summary.txt 2>&1
mkdir -p $out/keep
mv $out/full/binarysearch_inter_group.ncu-rep $out/keep/ 2>/dev/null
rm -f $out/full/*.ncu-rep
du -sh $out
