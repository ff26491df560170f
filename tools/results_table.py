"""Markdown results table from bench JSON lines (the suite's kernels, its
`rest10` kernels, and the extension variants).
usage: results_table.py FILE.json [FILE.json ...]"""
import json
import sys

VARS = ["intra_smem", "intra_reg", "inter_group"]
XV = ["inter_cluster", "intra_nolds", "dup_kernel"]
print("| config | kernel | bound | none ms | none frac of copy peak | " + " | ".join(VARS + XV) + " |")
print("|---|---|---|---|---|" + "---|" * (len(VARS) + len(XV)))
for f in sys.argv[1:]:
    d = json.loads(open(f).read().strip().splitlines()[-1])
    cfg = d["config"].get("preset", "?")
    xk = (d.get("extra_variants") or {}).get("kernels", {})
    rows = [(cfg, k, kv) for k, kv in d["kernels"].items()]
    rows += [("rest10", k, kv) for k, kv in (d.get("rest10") or {}).items() if isinstance(kv, dict)]
    for c, k, kv in rows:
        n = kv["none"]
        frac = f"{n['frac']:.2f}"
        if "tensor_frac" in n:
            frac = f"{n['tflops']:.0f} TFLOP/s = {n['tensor_frac']:.2f} of sustained bf16"
        cells = [f"{kv[v]['slowdown']:.2f}x" if v in kv else "" for v in VARS]
        cells += [f"{xk[k][v]['slowdown']:.2f}x" if k in xk and v in xk[k] else "" for v in XV]
        print(f"| {c} | {k} | {kv.get('bound', '')} | {n['ms']:.4g} | {frac} | " + " | ".join(cells) + " |")
