"""Instruction histograms of librmt's kernels from the local build's SASS
(cuobjdump -sass; no GPU needed): per kernel instantiation, the count of every
opcode, plus the tcgen05/TMA evidence (UTCHMMA, UTMALDG, LDTM, UTCBAR) for
MatMul.  usage: sass_hist.py OUT.json [object-file-substring ...]"""
import collections
import glob
import json
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
objs = sorted(glob.glob(os.path.join(ROOT, "paper_conf_isca_waddenlgss14_b200", "build", "k_*.o")))
only = sys.argv[2:]
out = {}
for o in objs:
    if only and not any(s in o for s in only):
        continue
    sass = subprocess.run(["cuobjdump", "-sass", o], capture_output=True, text=True).stdout
    cur = None
    for line in sass.splitlines():
        m = re.match(r"\s+Function : (\S+)", line)
        if m:
            cur = m.group(1)
            dem = subprocess.run(["c++filt", cur], capture_output=True, text=True).stdout.strip()
            # keep the template arguments <V, M> only: "k<1, 0>" style names
            short = re.sub(r"\(.*", "", dem.replace("rmt::(anonymous namespace)::", "").replace("void ", ""))
            cur = short
            out[cur] = collections.Counter()
            continue
        m = re.match(r"\s+/\*[0-9a-f]{4,}\*/\s+(@!?U?P\w+\s+)?([A-Z][A-Z0-9_.]*)", line)
        if m and cur:
            op = m.group(2).split(".")[0]
            out[cur][op] += 1
res = {k: dict(sorted(v.items(), key=lambda kv: -kv[1])) for k, v in out.items() if v}
with open(sys.argv[1], "w") as f:
    json.dump(res, f, indent=1)
for k, v in res.items():
    if "mm_kernel" in k:
        ev = {x: v.get(x, 0) for x in ("UTCHMMA", "UTCQMMA", "UTMALDG", "LDTM", "UTCBAR", "SYNCS")}
        print(k, "total", sum(v.values()), ev)
