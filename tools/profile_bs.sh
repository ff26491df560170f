#!/bin/bash
# BinarySearch evidence (run under gpurun from the repo root):
#   1. gather probe: DRAM bytes per random G-byte block read (G = 4..128)
#   2. ncu --set full of bins_kernel / bins_index_kernel (none, inter_group)
#   3. the launch list of a short default bench run
out=${1:-gpurun_out/bs}
mkdir -p $out
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -o /tmp/gp tools/gather_probe.cu && /tmp/gp > $out/gather.txt 2>&1
timeout 300 ncu --metrics dram__bytes_read.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_tex_op_read_lookup_miss.sum,gpu__time_duration.sum \
  --clock-control none -k regex:gather -s 15 -c 50 --csv /tmp/gp > $out/gather_ncu.csv 2>&1
for v in none inter_group; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:bins_ -c 2 -o $out/bins_$v \
    python tools/prof_run.py suite binarysearch $v 1 > $out/bins_$v.log 2>&1
  ncu -i $out/bins_$v.ncu-rep --page raw --csv > $out/bins_${v}_raw.csv 2>/dev/null
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $out/launches.csv \
  python bench.py --steps 2 --warmup 1 --no-cpu-baseline --e2e-steps 0 --energy-seconds 0 --extra-variants "" \
  --no-rest10 > $out/launches_bench.log 2>&1
python tools/launch_summary.py $out/launches.csv > $out/launches_summary.json 2>&1
ls -la $out
