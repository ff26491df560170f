"""Small launches of every kernel under every variant (for compute-sanitizer)."""
import sys, os
R = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, R); sys.path.insert(0, os.path.join(R, "tests"))
import numpy as np
from paper_conf_isca_waddenlgss14_b200 import rmt
from cases import (DCT, FWT, BinarySearch, BlackScholes, FloydWarshall, MatMul, PrefixSum, Reduction, Sobel,
                   Transpose)
from helpers import run
cases = [BlackScholes(3000), BinarySearch(5000, 1000), FWT(1 << 13), PrefixSum(4096 * 3 + 7), Reduction(100003),
         Transpose(68, 132), Sobel(37, 100), DCT(24, 264), FloydWarshall(52), MatMul(128, 256, 128)]
only = sys.argv[1:] or None
for c in cases:
    if only and c.kernel not in only:
        continue
    ref = None
    for v in ("none", "intra_smem", "intra_reg", "inter_group", "inter_cluster"):
        b = c.buffers()
        e = run(c.kernel, v, b, c.n, c.dims)
        o = c.outputs(b)
        ref = ref or o
        ok = e == 0 and all(np.array_equal(x, y) for x, y in zip(o, ref))
        print(c.kernel, v, "ok" if ok else f"MISMATCH err={e}", flush=True)
