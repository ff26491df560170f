import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_isca_waddenlgss14_b200 import rmt, workloads
j = workloads.job_binarysearch(1 << 26, 1 << 24)
b = j.device_buffers()
err = torch.zeros(1, dtype=torch.int64, device="cuda")
rmt.launch(j.kernel, "none", b, j.n, err, dims=j.dims); torch.cuda.synchronize()
ref = b[2].cpu().numpy().view(np.uint32).copy()
ws = rmt.make_workspace(j.kernel, "inter_group", j.n, j.dims)
for rep in range(3):
    err.zero_(); b[2].fill_(-1); torch.cuda.synchronize()
    t = time.time()
    rmt.launch(j.kernel, "inter_group", b, j.n, err, dims=j.dims, workspace=ws); torch.cuda.synchronize()
    dt = time.time() - t
    y = b[2].cpu().numpy().view(np.uint32)
    bad = np.nonzero(y != ref)[0]
    ctrl = ws[:16].cpu().numpy().view(np.uint32)
    print(f"rep{rep} t={dt:.3f}s err={int(err.item())} bad={bad.size} ctrl={ctrl[:4]}")
    if bad.size:
        lt = (bad // 4) % 256
        blk = bad // 1024
        print("  lane hist", np.bincount(lt % 32, minlength=32))
        print("  warp hist", np.bincount(lt // 32, minlength=8))
        print("  blocks", blk.min(), blk.max(), np.unique(blk).size, "sentinel", int((y[bad]==0xFFFFFFFF).sum()))
        # are whole warps bad?
        wb = bad // 128
        u, c = np.unique(wb, return_counts=True)
        print("  per-warp bad count hist", np.bincount(c)[:130:16])
