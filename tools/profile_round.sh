#!/bin/bash
# Round evidence on one B200 (run under gpurun from the repo root):
#   1. the ncu launch list of a short bench run   -> $out/launches.csv (+ launches_summary.json)
#   2. --set full captures of each suite kernel (and DCT, FloydWarshall pass,
#      MatMul, BlackScholes) under none / intra_smem / intra_reg / inter_group,
#      summarised on the box                       -> $out/ncu_full_summary.{json,txt}
# usage: tools/profile_round.sh [OUTDIR]
set -u
out=${1:-gpurun_out/prof}
mkdir -p $out/full
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $out/launches.csv \
  python bench.py --steps 2 --warmup 1 --no-cpu-baseline --e2e-steps 0 --energy-seconds 0 --extra-variants "" \
  --no-rest10 > $out/launches_bench.log 2>&1
python tools/launch_summary.py $out/launches.csv > $out/launches_summary.json 2>&1
# cfg kernel capture-name kernel-regex skip
for kv in "suite binarysearch binarysearch bins_kernel 1" "suite fwt fwt_p1 fwt_p1_kernel 1" "suite fwt fwt_ps fwt_ps_kernel 1" \
          "suite prefixsum prefixsum ps_scan_kernel 1" "suite reduction reduction red_partial_kernel 1" \
          "suite transpose transpose tr_kernel 1" "suite sobel sobel sobel_kernel 1" \
          "fwdct dct dct dct_kernel 1" "fwdct floydwarshall fw_pass fw_pass_kernel 300" \
          "mm8k matmul matmul mm_kernel 1" "bs30 blackscholes blackscholes bs_kernel 1"; do
  set -- $kv
  for vv in "none 0" "intra_smem 1" "intra_reg 2" "inter_group 3"; do
    set -- $kv $vv
    reps=2; [ "$2" = floydwarshall ] && reps=1
    regex="regex:$4<.int.$7, .int.0"
    skip=$5
    # FloydWarshall inter_group is one cooperative kernel (fw_coop_kernel) for all passes
    if [ "$2" = floydwarshall ] && [ "$6" = inter_group ]; then regex="regex:fw_coop_kernel<.int.3, .int.0"; skip=0; fi
    timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
      -k "$regex" -s $skip -c 1 -o $out/full/$3_$6 \
      python tools/prof_run.py $1 $2 $6 $reps > $out/full/$3_$6.log 2>&1
  done
done
ls -la $out $out/full
# summarise on the box (the .ncu-rep files together exceed gpurun's 64 MiB
# copy-back limit); keep the dominant kernel's report only
python tools/ncu_summary.py $out/full/*.ncu-rep --json $out/ncu_full_summary.json > $out/ncu_full_summary.txt 2>&1
python tools/traffic_from_summary.py $out/ncu_full_summary.json $out/ncu_traffic.json
mkdir -p $out/keep
mv $out/full/binarysearch_inter_group.ncu-rep $out/keep/ 2>/dev/null
rm -f $out/full/*.ncu-rep
du -sh $out
