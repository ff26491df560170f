"""Full-size false-alarm / bit-identity diagnostic: every job of a bench config,
every variant, err count and output diff vs none (run on the GPU box)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
from paper_conf_isca_waddenlgss14_b200 import rmt, workloads

cfg = sys.argv[1] if len(sys.argv) > 1 else "suite"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
for j in workloads.config_jobs(cfg):
    bufs = j.device_buffers()
    outs = [i for i, h in enumerate(j.host_in) if h is None]
    ref = None
    for v in ("none", "intra_smem", "intra_reg", "inter_group", "inter_cluster"):
        ws = rmt.make_workspace(j.kernel, v, j.n, j.dims)
        for r in range(reps):
            err = torch.zeros(1, dtype=torch.int64, device="cuda")
            for i in outs:
                bufs[i].fill_(-1)
            rmt.launch(j.kernel, v, bufs, j.n, err, dims=j.dims, workspace=ws)
            torch.cuda.synchronize()
            o = [bufs[i].clone() for i in outs]
            if ref is None:
                ref = o
            diff = sum(int((a != b).sum()) for a, b in zip(o, ref))
            print(f"{j.kernel:13s} {v:12s} rep{r} err={int(err.item())} diff_words={diff}", flush=True)
