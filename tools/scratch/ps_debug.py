"""Debug: PrefixSum partial words and first mismatch (none)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_isca_waddenlgss14_b200 import rmt, inputs
n = int(sys.argv[1]) if len(sys.argv) > 1 else 1 << 22
v = sys.argv[2] if len(sys.argv) > 2 else "none"
x = (inputs.u32(5, n, 0, stream=4) % np.uint32(256)).astype(np.uint32)
xd = torch.from_numpy(x.view(np.int32)).cuda()
y = torch.full((n,), -1, dtype=torch.int32, device="cuda")
err = torch.zeros(1, dtype=torch.int64, device="cuda")
ws = rmt.make_workspace("prefixsum", v, n)
rmt.launch("prefixsum", v, [xd, y], n, err, workspace=ws)
torch.cuda.synchronize()
ref = np.cumsum(x, dtype=np.uint64).astype(np.uint32)
got = y.cpu().numpy().view(np.uint32)
bad = np.nonzero(got != ref)[0]
print("err", int(err.item()), "nbad", bad.size, "first", bad[:5], got[bad[:5]] if bad.size else None, ref[bad[:5]] if bad.size else None)
w = ws.cpu().numpy()
ctl = w[:256].view(np.uint32)[:4]
part = w[256:256 + 8 * 2048].view(np.uint64)
print("ctl", ctl, "part[0:8]", [(int(p >> 32), int(p & 0xffffffff)) for p in part[:8]])
tile = 4096
print("expected tile sums", [int(x[t*tile:(t+1)*tile].sum()) for t in range(4)])
