"""Median device time per (kernel, variant) for a bench config (quick look).
usage: time_jobs.py CONFIG [REPS] [VARIANTS]   (RMT_KERNELS=a,b: only those kernels)"""
import sys, os, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_isca_waddenlgss14_b200 import rmt, workloads

cfg = sys.argv[1]
if os.environ.get("RMT_ABL"):  # full | nocomm | inflate
    rmt.set_ablation(os.environ["RMT_ABL"])
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 5
variants = sys.argv[3].split(",") if len(sys.argv) > 3 else ["none", "intra_smem", "intra_reg", "inter_group", "inter_cluster", "intra_nolds", "dup_kernel"]
only = os.environ.get("RMT_KERNELS", "").split(",") if os.environ.get("RMT_KERNELS") else None
for j in workloads.config_jobs(cfg):
    if only and j.kernel not in only:
        continue
    b = j.device_buffers()
    base = None
    for v in variants:
        ws = rmt.make_workspace(j.kernel, v, j.n, j.dims)
        err = torch.zeros(1, dtype=torch.int64, device="cuda")
        ts = []
        for r in range(reps + 1):
            if j.kernel == "floydwarshall":
                b[0].copy_(torch.from_numpy(j.host_in[0].view("int32").reshape(-1)).cuda())
            s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s.record()
            rmt.launch(j.kernel, v, b, j.n, err, dims=j.dims, workspace=ws)
            e.record()
            torch.cuda.synchronize()
            if r:
                ts.append(s.elapsed_time(e))
        ms = statistics.median(ts)
        base = base or ms
        extra = ""
        if j.kernel == "matmul":
            M, N, K = j.dims
            extra = f" {2*M*N*K/ms/1e9:.1f} TFLOP/s"
        else:
            extra = f" {j.alg_bytes/ms/1e6:.1f} GB/s"
        print(f"{j.kernel:13s} {v:12s} {ms:9.4f} ms  x{ms/base:5.2f}{extra} err={int(err.item())}", flush=True)
