"""Summarise an ncu --metrics gpu__time_duration.sum launch list: per kernel
(demangled name, template args) launch count, total and mean time, share."""
import csv, io, json, re, sys, collections

path = sys.argv[1]
txt = open(path).read()
start = txt.index('"ID"')
rows = list(csv.DictReader(io.StringIO(txt[start:])))
agg = collections.OrderedDict()
for r in rows:
    if r.get("Metric Name") != "gpu__time_duration.sum":
        continue
    name = r["Kernel Name"]
    m = re.search(r"(\w+_kernel)<([^>]*)>", name)
    key = f"{m.group(1)}<{m.group(2)}>" if m else name[:60]
    unit = r["Metric Unit"]
    v = float(r["Metric Value"].replace(",", ""))
    us = v * {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3}.get(unit, 1.0)
    a = agg.setdefault(key, [0, 0.0])
    a[0] += 1
    a[1] += us
tot = sum(v[1] for v in agg.values())
out = {k: {"launches": n, "total_us": round(t, 1), "mean_us": round(t / n, 2), "share": round(t / tot, 4)}
       for k, (n, t) in sorted(agg.items(), key=lambda kv: -kv[1][1])}
print(json.dumps({"total_us": round(tot, 1), "kernels": out}, indent=1))
