"""Inter-group CTA timeline from an RMT_TRACE experiment build (RMT_LIB=build_exp/trace.so):
per-CTA globaltimer milestones (Rep RMT_TR) -> phase durations per role.
usage: RMT_LIB=build_exp/trace.so python tools/trace_inter.py KERNEL_CONFIG"""
import ctypes
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_isca_waddenlgss14_b200 import rmt, workloads  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "suite:transpose"
L = rmt.lib()
L.rmt_trace_copy.argtypes = [ctypes.c_void_p, ctypes.c_size_t]
for j in workloads.config_jobs(cfg):
    b = j.device_buffers()
    ws = rmt.make_workspace(j.kernel, "inter_group", j.n, j.dims)
    err = torch.zeros(1, dtype=torch.int64, device="cuda")
    for _ in range(3):
        rmt.launch(j.kernel, "inter_group", b, j.n, err, dims=j.dims, workspace=ws)
    torch.cuda.synchronize()
    buf = np.zeros((1 << 17, 8), np.uint64)
    L.rmt_trace_copy(buf.ctypes.data, buf.nbytes)
    t = buf[buf[:, 0] > 0].astype(np.float64)
    t0 = t[:, 0].min()
    role = t[:, 7]
    print(f"{j.kernel}: {len(t)} CTAs, span {(t[:, 5].max() - t0) / 1e3:.1f} us")
    names = ["ticket+turn", "to 1st commit", "1st commit", "rest commits", "finish"]
    for r, nm in ((0, "producer"), (1, "consumer")):
        x = t[role == r]
        d = np.diff(x[:, :6], axis=1) / 1e3
        life = (x[:, 5] - x[:, 0]) / 1e3
        print(f"  {nm}: life med {np.median(life):.2f} us p90 {np.percentile(life, 90):.2f};",
              "; ".join(f"{n} {np.median(d[:, i]):.2f}/{np.percentile(d[:, i], 90):.2f}" for i, n in enumerate(names)))
    # pair start skew (consumer start - producer start), by ticket order
    rows = buf[: len(t)]
    st = rows[:, 0].astype(np.float64)
    npair = len(st) // 2
    skew = (st[1:2 * npair:2] - st[0:2 * npair:2]) / 1e3
    print(f"  pair start skew (cons - prod) med {np.median(skew):.2f} us p10 {np.percentile(skew, 10):.2f} "
          f"p90 {np.percentile(skew, 90):.2f}")
    # CTAs alive over time
    ev = np.concatenate([np.stack([t[:, 0], np.ones(len(t))], 1), np.stack([t[:, 5], -np.ones(len(t))], 1)])
    ev = ev[np.argsort(ev[:, 0], kind="stable")]
    alive = np.cumsum(ev[:, 1])
    print(f"  CTAs alive: median {np.median(alive):.0f} max {alive.max():.0f}")
