"""Run one kernel/variant of a bench config `reps` times (for ncu capture).
usage: prof_run.py CONFIG KERNEL VARIANT [REPS]"""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_isca_waddenlgss14_b200 import rmt, workloads

cfg, kern, var = sys.argv[1:4]
reps = int(sys.argv[4]) if len(sys.argv) > 4 else 2
j = [x for x in workloads.config_jobs(cfg) if x.kernel == kern][0]
b = j.device_buffers()
err = torch.zeros(1, dtype=torch.int64, device="cuda")
ws = rmt.make_workspace(j.kernel, var, j.n, j.dims)
torch.cuda.synchronize()
for _ in range(reps):
    rmt.launch(j.kernel, var, b, j.n, err, dims=j.dims, workspace=ws)
torch.cuda.synchronize()
print(kern, var, "err", int(err.item()), "launches/rep", rmt.last_launch_count())
