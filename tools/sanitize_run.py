"""Small launches of every kernel under every variant, for compute-sanitizer
(memcheck / racecheck / synccheck): each output checked bitwise against none.
  compute-sanitizer --tool memcheck python tools/sanitize_run.py [kernel ...]"""
import os
import sys

R = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, R)
sys.path.insert(0, os.path.join(R, "tests"))
import numpy as np  # noqa: E402

from paper_conf_isca_waddenlgss14_b200 import rmt  # noqa: E402
from cases import (DCT, DWT, FWT, BinarySearch, BinomialOption, BitonicSort, BlackScholes, BlackScholesIndep,  # noqa
                   FloydWarshall, MatMul, PrefixSum, Reduction, Sobel, Transpose)
from helpers import run  # noqa: E402

cases = [BlackScholes(3000), BlackScholesIndep(1024), BinarySearch(5000, 1000), BinarySearch(300000, 1000),
         BinarySearch(5000, 300, ghost=True), FWT(1 << 13), PrefixSum(4096 * 3 + 7),
         PrefixSum(4096 * 3 + 7, exclusive=True), PrefixSum(4096 * 3 + 7, f32=True),
         Reduction(100003), Transpose(68, 132), Sobel(37, 100), DCT(24, 264), FloydWarshall(52),
         MatMul(128, 256, 128), DWT(1 << 13), BitonicSort(1 << 13), BinomialOption(300)]
variants = ("none",) + rmt.RMT_VARIANTS
only = sys.argv[1:] or None
bad = 0
for c in cases:
    if only and c.kernel not in only:
        continue
    ref = None
    for stress in (False, True):
        for v in variants:
            if stress and v not in ("inter_group", "inter_cluster"):
                continue
            if stress:  # the queue stress instantiation: depth 1, tags, skew
                rmt.set_stress(1, rmt.STRESS_TAGS | rmt.STRESS_SKEW, 200, 0)
            b = c.buffers()
            e = run(c.kernel, v, b, c.n, c.dims)
            rmt.set_stress(0, 0, 0, 0)
            o = c.outputs(b)
            ref = ref or o
            ok = e == 0 and all(np.array_equal(x, y) for x, y in zip(o, ref))
            bad += not ok
            print(c.kernel, v + ("/stress" if stress else ""), "ok" if ok else f"MISMATCH err={e}", flush=True)
print("sanitize_run:", "all ok" if bad == 0 else f"{bad} mismatches")
