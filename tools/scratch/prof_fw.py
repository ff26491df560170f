"""Run FloydWarshall n=4096 once per variant (for ncu capture of individual passes)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_isca_waddenlgss14_b200 import rmt, workloads
var = sys.argv[1]
j = workloads.job_floydwarshall(4096)
b = j.device_buffers()
err = torch.zeros(1, dtype=torch.int64, device="cuda")
ws = rmt.make_workspace("floydwarshall", var, j.n)
rmt.launch("floydwarshall", var, b, j.n, err, workspace=ws)
torch.cuda.synchronize()
print(var, int(err.item()))
