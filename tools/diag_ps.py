import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle
from paper_conf_isca_waddenlgss14_b200 import rmt, workloads
n = 1 << 26
j = workloads.job_prefixsum(n)
x = j.host_in[0]
ref = oracle.prefixsum_u32(x)
b = j.device_buffers()
for mode in ["full", "nocomm", "full", "full"]:
    rmt.set_ablation(mode)
    ws = rmt.make_workspace("prefixsum", "inter_group", n)
    err = torch.zeros(1, dtype=torch.int64, device="cuda")
    b[1].fill_(-1)
    rmt.launch("prefixsum", "inter_group", b, n, err, workspace=ws)
    torch.cuda.synchronize()
    y = b[1].cpu().numpy().view(np.uint32)
    bad = np.nonzero(y != ref)[0]
    print(mode, "err", int(err.item()), "bad", bad.size)
    if bad.size:
        tiles = bad // 4096
        ltid = (bad % 4096) // 16
        print("  tiles", np.unique(tiles)[:20], "n_tiles", np.unique(tiles).size)
        print("  ltid", np.unique(ltid)[:40])
        print("  within-thread item", np.unique(bad % 16))
        d = (y[bad].astype(np.int64) - ref[bad].astype(np.int64)) % 2**32
        print("  delta", np.unique(d)[:10], "sentinel", int((y[bad] == 0xFFFFFFFF).sum()))
rmt.set_ablation("full")
