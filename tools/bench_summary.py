"""Print the headline numbers of a bench.py JSON line (file argument)."""
import json
import sys

d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
print("value", d["value"], "ms/step", d["ms_per_step"], "err", d["err_count"], "clocks", d["clocks"])
print("roofline", {k: d["roofline"][k] for k in ("kernel", "achieved", "frac", "share_of_step")})
for v, g in d["slowdown_geomean"].items():
    print("geomean", v, {k: g[k] for k in ("config", "all10", "mem_subset")})
allk = dict(d["kernels"])
allk.update({k: x for k, x in (d.get("rest10") or {}).items() if isinstance(x, dict)})
for k, x in allk.items():
    row = {v: (x[v]["ms"] if v == "none" else x[v]["slowdown"]) for v in x if isinstance(x[v], dict)}
    print(f"{k:14s}", row, "frac", x["none"]["frac"])
if d.get("extra_variants"):
    print("extra", d["extra_variants"]["slowdown_geomean"])
    for k, x in d["extra_variants"]["kernels"].items():
        print(f"  {k:14s}", {v: x[v]["slowdown"] for v in x})
