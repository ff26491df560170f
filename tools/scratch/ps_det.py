import sys; import os; R=os.path.dirname(os.path.dirname(os.path.abspath(__file__))); sys.path.insert(0,R); sys.path.insert(0,R+'/tests')
import numpy as np, torch
from paper_conf_isca_waddenlgss14_b200 import rmt
from cases import PrefixSum
from helpers import run
import oracle
c = PrefixSum(4096 * 9 + 5)
ref = oracle.prefixsum_u32(c.x)
def go(f=None):
    if f: rmt.inject_fault(*f)
    try:
        b = c.buffers(); e = run("prefixsum", "none", b, c.n); return e, c.outputs(b)[0]
    finally:
        rmt.clear_faults()
bad = 0
for i in range(20):
    e, o = go(); bad += not np.array_equal(o, ref)
print("normal runs wrong:", bad)
for i in range(5):
    e, o = go((0, "smem", 22, 1362)); d = np.nonzero(o != ref)[0]
    print("fault run: err", e, "diff", d.size, d[:5], (d // 4096)[:5] if d.size else None)
for i in range(3):
    e, o = go((0, "smem", 22, 10**9)); print("fault(no-match) diff", np.sum(o != ref))
