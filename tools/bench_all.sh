#!/bin/bash
# Bench lines for every BASELINE.json config (run under gpurun from the repo root):
#   gpurun_out/benches/<config>.json, plus the suite with the cost-attribution
#   ablations (INFLATE / NOCOMM) as suite_ablations.json.
out=gpurun_out/benches
mkdir -p $out
for c in suite bs16 suite28 fwdct bs30 mm16k comm; do
  timeout 900 python bench.py --config $c > $out/$c.log 2>&1
  grep '^{' $out/$c.log | tail -1 > $out/$c.json
done
timeout 900 python bench.py --ablations --extra-variants "" > $out/suite_ablations.log 2>&1
grep '^{' $out/suite_ablations.log | tail -1 > $out/suite_ablations.json
ls -la $out
