#!/usr/bin/env python
"""bench.py -- RMT slowdown per variant and baseline HBM GB/s vs peak
(BASELINE.json metric) on the APP SDK-style suite (BASELINE.json configs[1]).

One step = one pass of the whole hot path over one batch of synthetic input:
every kernel of the config launched once under each variant
(none, intra_smem, intra_reg, inter_group) through the C ABI (librmt.so).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config suite] [--impl rmt|reference]

value      = the unprotected baseline's aggregate HBM GB/s over the config's kernels:
             sum of their algorithmic bytes / sum of their `none` launch times
             (CUDA events inside the timed region, max over ranks; the metric's
             "baseline HBM GB/s"); inputs resident in HBM, every input > L2.
slowdown   = per kernel t(variant) / t(none) (median launch time), and the geomean
             per variant over the config, over all ten BASELINE.json kernels
             (the configs[1] suite timed in the step + BlackScholes 2^30,
             FloydWarshall 4096, DCT 8192^2, MatrixMultiplication 16384^3 timed
             after it) and over SURVEY's memory-bound subset.
e2e        = the same baseline metric through rmt_run_host_variants (pinned host
             buffers; per kernel one H2D of its inputs, the four variants, one D2H
             of the committed outputs and error counts, inside the timed region).
The reference arm (--impl reference) is the CPU oracle (oracle/), timed as it
stands on this host's cores on a bounded sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import platform
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "RMT slowdown vs unprotected kernel per variant; baseline HBM GB/s vs peak"
VARIANTS = ("none", "intra_smem", "intra_reg", "inter_group")
# B200 extensions: measured after the timed step, not part of it
EXTRA_VARIANTS = ("inter_cluster", "intra_nolds", "dup_kernel")
SPEC_HBM_GBS = 8000.0  # BASELINE.json north_star "~8 TB/s" (the >= 70 % target is vs 8 TB/s)


# ---------------------------------------------------------------- energy (NVML; Fig. 5)
def measure_energy(dev_index, launch, seconds=0.25):
    """Back-to-back launches for >= `seconds`: average board power (W) from the
    NVML total-energy counter (mJ) over the device time, and energy per launch."""
    import torch
    try:
        import pynvml
        pynvml.nvmlInit()
        h = pynvml.nvmlDeviceGetHandleByIndex(dev_index)
        pynvml.nvmlDeviceGetTotalEnergyConsumption(h)
    except Exception:
        return None
    launch()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    launch()
    torch.cuda.synchronize()
    one = max(time.perf_counter() - t0, 1e-5)
    reps = max(3, int(seconds / one))
    e0 = pynvml.nvmlDeviceGetTotalEnergyConsumption(h)
    a = torch.cuda.Event(enable_timing=True)
    b = torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps):
        launch()
    b.record()
    torch.cuda.synchronize()
    e1 = pynvml.nvmlDeviceGetTotalEnergyConsumption(h)
    secs = a.elapsed_time(b) * 1e-3
    joules = (e1 - e0) * 1e-3
    return {"avg_w": round(joules / secs, 1), "j_per_launch": round(joules / reps, 6), "launches": reps,
            "ms_per_launch": round(1e3 * secs / reps, 4)}


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=10)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--config", default="suite")
    p.add_argument("--impl", default="rmt", choices=["rmt", "reference"])
    p.add_argument("--e2e-steps", type=int, default=2)
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--no-rest10", action="store_true",
                   help="skip the four other BASELINE.json kernels (all-10 slowdown geomean)")
    p.add_argument("--variants", default=",".join(VARIANTS))
    p.add_argument("--extra-variants", default=",".join(EXTRA_VARIANTS),
                   help="variants timed per launch after the timed region (reported, not in the step)")
    p.add_argument("--energy-seconds", type=float, default=0.25,
                   help="per (kernel, variant) NVML energy window; 0 disables the energy table")
    p.add_argument("--ablations", action="store_true",
                   help="also time the INFLATE and NOCOMM ablations per kernel x RMT variant (cost attribution)")
    p.add_argument("--fwt-exchange", default="p2p", choices=["p2p", "sendrecv"],
                   help="multi-GPU FWT cross-shard stage: the fused combine kernel reading the partner's shard over "
                        "NVLink peer memory (p2p), or NCCL send/recv then the combine kernel")
    p.add_argument("--dist-backend", default="nccl",
                   help="nccl (one GPU per rank); gloo only to exercise the multi-rank path on one GPU")
    return p.parse_args()


def load_peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(path) as f:
            pk = json.load(f)
        return float(pk["hbm_gbs"]), "measured copy (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md)"


def load_tensor_peak():
    """Dense bf16 TFLOP/s: the SUSTAINED measured figure (a matmul launch sits
    inside a long step of back-to-back launches), else the guide's fallback."""
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            pk = json.load(f)
        return float(pk["bf16_tflops_sustained"]), "measured sustained bf16 (MEASURED_PEAKS.json)"
    except Exception:
        return 2250.0 * 0.75, "fallback (B200_PROFILING.md nominal x 0.75)"


def job_flops(j):
    if j.kernel == "matmul":
        M, N, K = j.dims
        return 2.0 * M * N * K
    return None


def load_traffic():
    path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        with open(path) as f:
            return json.load(f)
    except Exception:
        return {}


def geomean(xs):
    xs = [x for x in xs if x and x > 0]
    return round(math.exp(sum(math.log(x) for x in xs) / len(xs)), 3) if xs else None


# ---------------------------------------------------------------- clocks (NVML, sampled during the timed region)
class ClockSampler:
    REASONS = {0x4: "sw_power_cap", 0x8: "hw_slowdown", 0x20: "sw_thermal_slowdown",
               0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown"}

    def __init__(self, dev_index):
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self._stop = threading.Event()
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(dev_index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.nv = None

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for bit, name in self.REASONS.items():
                    if r & bit:
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(0.05)

    def __enter__(self):
        if self.nv:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        if self.nv:
            self._stop.set()
            self.t.join()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons)}
        return {"sm_mhz": statistics.median(self.samples), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


# ---------------------------------------------------------------- CPU oracle (reference arm / cpu_baseline)
def cpu_model():
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return platform.processor() or platform.machine()


def oracle_call(j, frac=1.0):
    """(callable, units, description) timing the oracle on job j, on the first
    `frac` of its units (frac = 1: the full config size; rows/elements taken from
    the job's own host inputs)."""
    import numpy as np

    import oracle
    if j.kernel == "binarysearch":
        A, q = j.host_in[0], j.host_in[1]
        q = q[: max(1, int(q.size * frac))]
        return (lambda: oracle.binarysearch(A, q)), q.size, f"binarysearch Q={q.size} on N={A.size}"
    if j.kernel == "fwt":
        m = max(1, int(j.n * frac))
        m = 1 << (m.bit_length() - 1)
        x = j.host_in[0][:m]
        return (lambda: oracle.fwt_f64(x)), x.size, f"fwt N={m}"
    if j.kernel in ("prefixsum", "reduction"):
        x = j.host_in[0][: max(1, int(j.n * frac))]
        fn = oracle.prefixsum_u32 if j.kernel == "prefixsum" else oracle.reduction_u32
        return (lambda: fn(x)), x.size, f"{j.kernel} n={x.size}"
    if j.kernel == "transpose":
        H, W = j.dims
        h = max(4, int(H * frac))
        A = np.ascontiguousarray(j.host_in[0].reshape(H, W)[:h])
        return (lambda: oracle.transpose_u32(A)), A.size, f"transpose {h}x{W}"
    if j.kernel == "sobel":
        H, W = j.dims
        h = max(3, int(H * frac))
        I = np.ascontiguousarray(j.host_in[0].reshape(H, W)[:h]).view(np.uint8).reshape(h, W, 4)
        return (lambda: oracle.sobel(I)), h * W, f"sobel {h}x{W}"
    if j.kernel == "blackscholes":
        m = max(1, int(j.n * frac))
        if j.host_in[0] is not None:
            r = j.host_in[0][:m]
        else:  # inputs generated in HBM (2^30 options): a bounded host sample of the same draws
            from paper_conf_isca_waddenlgss14_b200 import inputs
            m = min(m, 1 << 25)
            r = inputs.blackscholes_r(1, m)
        return (lambda: oracle.blackscholes(r)), r.size, f"blackscholes n={r.size}"
    if j.kernel == "matmul":  # a bounded block of C (1024 x 1024 outputs at frac 1) over the full K
        from paper_conf_isca_waddenlgss14_b200 import inputs
        M, N, K = j.dims
        m = max(1, min(M, max(64, int(1024 * frac))))
        n = max(1, min(N, max(64, int(1024 * frac))))
        A = j.host_in[0][: m * K].reshape(m, K) if j.host_in[0] is not None else inputs.matmul_bf16_normal(10, m, K, 22)
        Bt = j.host_in[1][: n * K].reshape(n, K) if j.host_in[1] is not None else inputs.matmul_bf16_normal(10, n, K, 24)
        return (lambda: oracle.matmul_bf16(A, Bt)), m * n, f"matmul {m}x{n}x{K} block"
    if j.kernel == "dwthaar1d":
        m = max(1, int(j.n * frac))
        m = 1 << (m.bit_length() - 1)
        x = j.host_in[0][:m]
        return (lambda: oracle.dwthaar1d_f64(x)), x.size, f"dwthaar1d N={m}"
    if j.kernel == "bitonicsort":
        x = j.host_in[0][: max(1, int(j.n * frac))]
        return (lambda: oracle.sort_u32(x)), x.size, f"sort n={x.size}"
    if j.kernel == "binomialoption":
        r = j.host_in[0][: max(1, min(j.n, 1 << 14, int(j.n * frac)))]
        return (lambda: oracle.binomialoption(r)), r.size, f"binomialoption n={r.size}"
    if j.kernel == "dct":
        H, W = j.dims
        h = max(8, int(H * frac) // 8 * 8)
        X = np.ascontiguousarray(j.host_in[0].reshape(H, W)[:h])
        return (lambda: oracle.dct8x8(X)), h * W, f"dct {h}x{W}"
    return None


def oracle_rate(jobs, frac=1.0, threads=None):
    """Time the oracle as it stands on every job (one run each at `frac` of the
    config size): returns (baseline-equivalent GB/s, seconds, cores, description).
    Units are converted with each job's algorithmic bytes per unit, so the rate
    is the GPU line's `value` measure."""
    import oracle
    if threads:
        oracle.set_threads(threads)
    try:
        tot_b = tot_s = 0.0
        desc = []
        for j in jobs:
            c = oracle_call(j, frac)
            if c is None:
                continue
            fn, units, what = c
            t0 = time.perf_counter()
            fn()
            dt = time.perf_counter() - t0
            tot_b += units * (j.alg_bytes / j.n)
            tot_s += dt
            desc.append(f"{what} {dt:.2f}s")
        if tot_s <= 0.0:
            return None, 0.0, oracle.num_threads(), "no oracle sample for this config"
        return tot_b / tot_s / 1e9, tot_s, oracle.num_threads(), "; ".join(desc)
    finally:
        if threads:
            oracle.set_threads(os.cpu_count() or 1)


# ---------------------------------------------------------------- reference arm
def reference_arm(args, rank):
    if rank != 0:
        return  # rank 0 alone runs the CPU reference arm
    from paper_conf_isca_waddenlgss14_b200 import workloads
    jobs = workloads.config_jobs(args.config, 0)
    frac = 1.0 / 16  # each step: a bounded 1/16 sample of every kernel of the config
    for _ in range(args.warmup):
        oracle_rate(jobs, frac / 4)
    rates, times = [], []
    desc, cores = "", 0
    for _ in range(args.steps):
        rate, secs, cores, desc = oracle_rate(jobs, frac)
        rates.append(rate)
        times.append(secs)
    rate = statistics.median(rates)
    line = {
        "impl": "reference", "metric": METRIC, "value": round(rate, 3), "unit": "GB/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round(1e3 * statistics.mean(times), 3), "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "u32/f32/u8x4", "data": "synthetic",
        "config": {"workload": workloads.CONFIG_TITLES[args.config], "preset": args.config},
        "cpu_baseline": {"value": round(rate, 3), "unit": "GB/s", "cores": cores, "kind": "oracle",
                         "sample": f"1/16 of every kernel per step: {desc}", "cpu": cpu_model()},
        "e2e": {"value": round(rate, 3), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------- main
def main():
    args = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        return reference_arm(args, rank)

    import torch
    import torch.distributed as dist

    from paper_conf_isca_waddenlgss14_b200 import parallel, rmt, workloads

    dev_index = local_rank % max(1, torch.cuda.device_count())
    torch.cuda.set_device(dev_index)
    if world > 1:
        if args.dist_backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", dev_index))
        else:
            dist.init_process_group(args.dist_backend)
    variants = [v for v in args.variants.split(",") if v]
    jobs = workloads.config_jobs(args.config, rank, world)
    scaling = "strong" if args.config in workloads.STRONG_CONFIGS else "weak"
    stream = torch.cuda.current_stream()
    err = torch.zeros(1, dtype=torch.int64, device="cuda")
    ws = {}
    ws_aux = {}
    for j in jobs:
        j.device_buffers()
        for v in variants:
            ws[(j.kernel, v)] = rmt.make_workspace(j.kernel, v, j.n, j.dims)
            if world > 1 and j.kernel == "prefixsum":
                ws_aux[(j.kernel, v)] = rmt.make_workspace("reduction", v, j.n)
            if world > 1 and j.kernel == "fwt":
                ws_aux[(j.kernel, v)] = rmt.make_workspace("fwt", v, j.n, (1, 0))
    torch.cuda.synchronize()

    launches = [(j, v) for j in jobs for v in variants]
    ev = {(j.kernel, v): [] for j, v in launches}
    counts = {"gpu_launches": 0}
    # multi-GPU exchange buffers: PrefixSum totals, FWT partner shard
    s_tmp = torch.zeros(2, dtype=torch.int32, device="cuda")
    totals = torch.zeros(world, dtype=torch.int64, device="cuda")
    fwt_n = max([j.n for j in jobs if j.kernel == "fwt"] or [0])
    fwt_recv = torch.empty(fwt_n if world > 1 and args.fwt_exchange == "sendrecv" else 0, dtype=torch.float32,
                           device="cuda")
    fwt_tmp = torch.empty_like(fwt_recv)
    peer_fwt = parallel.PeerFWT(fwt_n, rmt) if world > 1 and fwt_n and args.fwt_exchange == "p2p" else None

    def one(j, v):
        """One launch of job j under variant v; for N > 1 the kernels that need a
        cross-shard exchange do it here (parallel.py)."""
        if world > 1 and j.kernel == "prefixsum":
            # local total (Reduction kernel) -> device all-gather -> device carry -> scan
            return parallel.global_prefixsum(j.dev[0], j.dev[1], s_tmp, totals, err, rmt, variant=v,
                                             ws_red=ws_aux[(j.kernel, v)], ws_ps=ws[(j.kernel, v)]) + 1
        if world > 1 and j.kernel == "fwt":
            # local transform + log2 G cross-shard butterfly stages: the combine kernel reads the
            # partner's shard over peer memory (fused), or after an NCCL send/recv
            if peer_fwt is not None:
                return peer_fwt.run(j.dev[0], err, v, workspace=ws[(j.kernel, v)], ws_comb=ws_aux[(j.kernel, v)])[1]
            return parallel.global_fwt(j.dev[0], j.dev[1].view(torch.float32), fwt_recv, fwt_tmp, err, rmt,
                                       variant=v, workspace=ws[(j.kernel, v)], ws_comb=ws_aux[(j.kernel, v)])
        if world > 1 and j.kernel == "reduction":
            rmt.launch(j.kernel, v, j.dev, j.n, err, dims=j.dims, workspace=ws[(j.kernel, v)],
                       stream=stream.cuda_stream)
            parallel.allreduce_sum_(j.dev[1].view(torch.int64))
            return rmt.last_launch_count()
        return rmt.launch(j.kernel, v, j.dev, j.n, err, dims=j.dims, workspace=ws[(j.kernel, v)],
                          stream=stream.cuda_stream)

    def step(timed):
        for j, v in launches:
            if timed:
                a = torch.cuda.Event(enable_timing=True)
                b = torch.cuda.Event(enable_timing=True)
                a.record(stream)
            nk = one(j, v)
            if timed:
                b.record(stream)
                ev[(j.kernel, v)].append((a, b))
                counts["gpu_launches"] += nk

    for _ in range(args.warmup):
        step(False)
    torch.cuda.synchronize()
    err.zero_()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    t0 = torch.cuda.Event(enable_timing=True)
    t1 = torch.cuda.Event(enable_timing=True)
    with ClockSampler(dev_index) as clk:
        t0.record(stream)
        for _ in range(args.steps):
            step(True)
        t1.record(stream)
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    ms_total = t0.elapsed_time(t1)
    # device time of every `none` launch in the timed region (the baseline metric)
    none_ms = sum(a.elapsed_time(b) for (k, v), lst in ev.items() if v == "none" for a, b in lst)
    if world > 1:
        tt = torch.tensor([ms_total, none_ms], dtype=torch.float64, device="cuda")
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        ms_total, none_ms = float(tt[0].item()), float(tt[1].item())
        parallel.allreduce_sum_(err)  # error counters of every rank, once for the whole timed region
    errs = int(err.item())

    # per-launch device times
    per = {(k, v): statistics.median(a.elapsed_time(b) for a, b in lst) for (k, v), lst in ev.items()}
    peak, peak_src = load_peaks()
    none_bytes = sum(j.alg_bytes for j in jobs) if "none" in variants else 0
    value = none_bytes * args.steps * world / (none_ms * 1e-3) / 1e9 if none_ms else None
    step_bytes = sum(j.alg_bytes for j, _ in launches)

    kernels = {}
    for j in jobs:
        d = {"bound": j.bound}
        for v in variants:
            ms = per[(j.kernel, v)]
            gbs = j.alg_bytes / (ms * 1e-3) / 1e9
            d[v] = {"ms": round(ms, 4), "gbs": round(gbs, 1), "frac": round(gbs / peak, 4)}
            if job_flops(j):
                tf = job_flops(j) / (ms * 1e-3) / 1e12
                d[v]["tflops"] = round(tf, 1)
                d[v]["tensor_frac"] = round(tf / load_tensor_peak()[0], 4)
            if v != "none" and "none" in variants:
                d[v]["slowdown"] = round(ms / per[(j.kernel, "none")], 3)
        kernels[j.kernel] = d

    # ---- configs[0] (BlackScholes 2^16, launch-latency bound): microseconds per
    # launch from a CUDA graph of 100 launches per variant (SURVEY.md:559)
    graph_us = None
    if args.config == "bs16":
        graph_us = {}
        err_g = torch.zeros(1, dtype=torch.int64, device="cuda")
        gs = torch.cuda.Stream()
        for j in jobs:
            for v in variants:
                w = ws[(j.kernel, v)]
                gs.wait_stream(stream)
                with torch.cuda.stream(gs):
                    for _ in range(3):  # warm outside the capture (lazy module loading)
                        rmt.launch(j.kernel, v, j.dev, j.n, err_g, dims=j.dims, workspace=w, stream=gs.cuda_stream)
                    g = torch.cuda.CUDAGraph()
                    with torch.cuda.graph(g, stream=gs):
                        for _ in range(100):
                            rmt.launch(j.kernel, v, j.dev, j.n, err_g, dims=j.dims, workspace=w,
                                       stream=gs.cuda_stream)
                stream.wait_stream(gs)
                ts = []
                for r in range(6):
                    a = torch.cuda.Event(enable_timing=True)
                    b = torch.cuda.Event(enable_timing=True)
                    a.record(stream)
                    g.replay()
                    b.record(stream)
                    torch.cuda.synchronize()
                    if r:
                        ts.append(a.elapsed_time(b) * 1e3 / 100)
                graph_us[v] = round(statistics.median(ts), 3)
                del g
        graph_us = {"us_per_launch": graph_us, "note": "median of 5 replays of a CUDA graph of 100 launches",
                    "slowdown": {v: round(graph_us[v] / graph_us["none"], 3) for v in graph_us if "none" in graph_us},
                    "err_count": int(err_g.item())}

    # ---- the four other BASELINE.json kernels (per-launch medians after the step)
    rest = {}
    if not args.no_rest10 and args.config == "suite" and "none" in variants:
        err_r = torch.zeros(1, dtype=torch.int64, device="cuda")
        for j in workloads.config_jobs("rest10", rank, world):
            j.device_buffers()
            d = {"bound": j.bound}
            for v in variants:
                w = rmt.make_workspace(j.kernel, v, j.n, j.dims)
                reps = 2 if j.kernel == "floydwarshall" and v == "inter_group" else 3
                ts = []
                for r in range(reps + 1):
                    if j.kernel == "floydwarshall":  # D is in/out: every launch restarts from W
                        j.dev[0].copy_(torch.from_numpy(j.host_in[0].view("int32").reshape(-1)).cuda())
                    a = torch.cuda.Event(enable_timing=True)
                    b = torch.cuda.Event(enable_timing=True)
                    a.record(stream)
                    rmt.launch(j.kernel, v, j.dev, j.n, err_r, dims=j.dims, workspace=w, stream=stream.cuda_stream)
                    b.record(stream)
                    torch.cuda.synchronize()
                    if r:
                        ts.append(a.elapsed_time(b))
                ms = statistics.median(ts)
                gbs = j.alg_bytes / (ms * 1e-3) / 1e9
                d[v] = {"ms": round(ms, 4), "gbs": round(gbs, 1), "frac": round(gbs / peak, 4)}
                if job_flops(j):
                    tf = job_flops(j) / (ms * 1e-3) / 1e12
                    d[v]["tflops"] = round(tf, 1)
                    d[v]["tensor_frac"] = round(tf / load_tensor_peak()[0], 4)
                del w
            for v in variants:
                if v != "none":
                    d[v]["slowdown"] = round(d[v]["ms"] / d["none"]["ms"], 3)
            d["mem_subset"] = j.mem_subset
            rest[j.kernel] = d
            j.dev = None
            torch.cuda.empty_cache()
        rest["err_count"] = int(err_r.item())

    all_k = dict(kernels)
    all_k.update({k: d for k, d in rest.items() if isinstance(d, dict)})
    mem_kernels = {"reduction", "transpose", "sobel", "prefixsum", "fwt", "dct"}
    slowdown_geomean = {}
    for v in variants:
        if v == "none":
            continue
        slowdown_geomean[v] = {
            "config": geomean([kernels[k][v]["slowdown"] for k in kernels]),
            "all10": geomean([all_k[k][v]["slowdown"] for k in all_k]) if rest else None,
            "mem_subset": geomean([all_k[k][v]["slowdown"] for k in all_k if k in mem_kernels]),
            "kernels": sorted(all_k),
        }
    baseline_frac = {}
    for k, d in all_k.items():
        if "none" not in d:
            continue
        g = d["none"]["gbs"]
        e = {"gbs": g, "vs_8tbps": round(g / SPEC_HBM_GBS, 4), "vs_copy_peak": round(g / peak, 4),
             "bound": d["bound"], "target_applies": k in mem_kernels}
        if "tflops" in d["none"]:
            e["tflops"] = d["none"]["tflops"]
            e["tensor_frac"] = d["none"]["tensor_frac"]
        baseline_frac[k] = e

    # dominant kernel (largest share of the step) -> roofline
    dj, dv = max(launches, key=lambda jv: per[(jv[0].kernel, jv[1])])
    dms = per[(dj.kernel, dv)]
    ach = dj.alg_bytes / (dms * 1e-3) / 1e9
    traffic = load_traffic().get(f"{dj.kernel}/{dv}")
    roofline = {"bound": "hbm", "achieved": round(ach, 1), "peak": peak, "unit": "GB/s",
                "frac": round(ach / peak, 4), "traffic": traffic, "kernel": f"{dj.kernel}/{dv}",
                "kernel_bound_class": dj.bound,
                "share_of_step": round(dms * args.steps / ms_total, 3), "peak_source": peak_src,
                "algorithmic_bytes_per_launch": dj.alg_bytes, "bytes_per_unit": round(dj.alg_bytes / dj.n, 3),
                "units_per_launch": dj.n}
    if dj.bound == "tensor" and job_flops(dj):
        tpk, tsrc = load_tensor_peak()
        tach = job_flops(dj) / (dms * 1e-3) / 1e12
        roofline.update({"bound": "tensor", "achieved": round(tach, 1), "peak": tpk, "unit": "TFLOP/s",
                         "frac": round(tach / tpk, 4), "peak_source": tsrc,
                         "algorithmic_flops_per_launch": job_flops(dj)})

    # ---- end to end through the public C ABI with host buffers
    e2e = None
    if args.e2e_steps > 0 and all(j.host_inputs for j in jobs):
        hosts = {j.kernel: j.pinned_host() for j in jobs}
        err_d = {j.kernel: torch.zeros(len(variants), dtype=torch.int64, device="cuda") for j in jobs}
        err_h = {j.kernel: torch.zeros(len(variants), dtype=torch.int64).pin_memory() for j in jobs}
        wsl = {j.kernel: [ws[(j.kernel, v)] for v in variants] for j in jobs}
        # rmt_run_host_variants_pipelined: inputs on one copy stream, every launch
        # on ONE compute stream (the kernels stay serialised), outputs on a second
        # copy stream, so the next kernel's H2D and the previous one's D2H overlap
        # the current kernel's variants (the two copy engines run concurrently)
        s_h2d, s_d2h = torch.cuda.Stream(), torch.cuda.Stream()

        def e2e_step():
            hb = db = 0
            # a step's input copies start after the previous step's launches: a
            # kernel's device inputs (FloydWarshall's D is in/out) are not
            # overwritten while its previous call still runs
            s_h2d.wait_stream(stream)
            for j in jobs:
                h, d_ = rmt.run_host_variants_pipelined(j.kernel, variants, hosts[j.kernel], j.dev, j.n,
                                                        err_d[j.kernel], wsl[j.kernel], err_h[j.kernel],
                                                        (s_h2d, stream, s_d2h), dims=j.dims)
                hb += h
                db += d_
            return hb, db

        def e2e_errors():
            return sum(int(x) for j in jobs for x in err_h[j.kernel].tolist())

        e2e_step()  # warm
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        h2d = d2h = e2e_err = 0
        e0.record(stream)
        s_h2d.wait_event(e0)
        s_d2h.wait_event(e0)
        for _ in range(args.e2e_steps):
            hb, db = e2e_step()
            h2d += hb
            d2h += db
        stream.wait_stream(s_h2d)
        stream.wait_stream(s_d2h)
        e1.record(stream)
        torch.cuda.synchronize()
        e2e_err = e2e_errors()  # the last step's counts (every step launches the same work)
        ems = e0.elapsed_time(e1)
        if world > 1:
            tt = torch.tensor([ems], dtype=torch.float64, device="cuda")
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
            ems = float(tt.item())
        # the baseline metric end to end: the unprotected bytes over the wall of the
        # whole host-buffer step (copies + every variant)
        e2e = {"value": round(none_bytes * args.e2e_steps * world / (ems * 1e-3) / 1e9, 3), "unit": "GB/s",
               "h2d_bytes_per_step": h2d // args.e2e_steps, "d2h_bytes_per_step": d2h // args.e2e_steps,
               "ms_per_step": round(ems / args.e2e_steps, 3), "err_count": e2e_err,
               "note": "per kernel: one H2D of its inputs, the variants, one D2H of the committed outputs and "
                       "error counts (rmt_run_host_variants_pipelined: H2D / compute / D2H on three streams, "
                       "consecutive kernels overlap; the launches stay serialised on one compute stream)"}

    # ---- cost attribution "as the paper does"
    attribution = None
    if args.ablations:
        attribution = {}
        for j in jobs:
            d = {}
            for v in [x for x in variants if x != "none"]:
                row = {}
                for mode in ("inflate", "nocomm", "full"):
                    rmt.set_ablation(mode)
                    ts = []
                    for r in range(4):
                        a = torch.cuda.Event(enable_timing=True)
                        b = torch.cuda.Event(enable_timing=True)
                        a.record(stream)
                        rmt.launch(j.kernel, v, j.dev, j.n, err, dims=j.dims, workspace=ws[(j.kernel, v)],
                                   stream=stream.cuda_stream)
                        b.record(stream)
                        torch.cuda.synchronize()
                        if r:
                            ts.append(a.elapsed_time(b))
                    row[mode] = statistics.median(ts)
                rmt.set_ablation("full")
                base = per[(j.kernel, "none")]
                row = {k: round(x, 4) for k, x in row.items()}
                row["scheduling"] = round(row["inflate"] / base - 1, 3)
                row["redundant_compute"] = round((row["nocomm"] - row["inflate"]) / base, 3)
                row["communication"] = round((row["full"] - row["nocomm"]) / base, 3)
                d[v] = row
            attribution[j.kernel] = d
        err.zero_()

    # ---- B200-native extension variants: per-launch medians outside the timed step
    extra = None
    xvars = [v for v in args.extra_variants.split(",") if v and v not in variants]
    if xvars and "none" in variants:
        extra = {"kernels": {}, "slowdown_geomean": {}}
        xs = {v: [] for v in xvars}
        err_x = torch.zeros(1, dtype=torch.int64, device="cuda")
        for j in jobs:
            d = {}
            for v in xvars:
                wsx = rmt.make_workspace(j.kernel, v, j.n, j.dims)
                ts = []
                for r in range(5):
                    a = torch.cuda.Event(enable_timing=True)
                    b = torch.cuda.Event(enable_timing=True)
                    a.record(stream)
                    rmt.launch(j.kernel, v, j.dev, j.n, err_x, dims=j.dims, workspace=wsx, stream=stream.cuda_stream)
                    b.record(stream)
                    torch.cuda.synchronize()
                    if r:
                        ts.append(a.elapsed_time(b))
                ms = statistics.median(ts)
                sd = ms / per[(j.kernel, "none")]
                d[v] = {"ms": round(ms, 4), "slowdown": round(sd, 3)}
                xs[v].append(sd)
                del wsx
            extra["kernels"][j.kernel] = d
        extra["slowdown_geomean"] = {v: geomean(s_) for v, s_ in xs.items()}
        extra["err_count"] = int(err_x.item())

    # ---- average power and energy per launch for every kernel x variant
    energy = None
    if args.energy_seconds > 0 and world == 1:
        energy = {}
        allv = variants + [v for v in args.extra_variants.split(",") if v and v not in variants]
        err_e = torch.zeros(1, dtype=torch.int64, device="cuda")
        for j in jobs:
            d = {}
            for v in allv:
                wsx = ws.get((j.kernel, v))
                if wsx is None:
                    wsx = rmt.make_workspace(j.kernel, v, j.n, j.dims)
                r = measure_energy(dev_index, lambda: rmt.launch(j.kernel, v, j.dev, j.n, err_e, dims=j.dims,
                                                                 workspace=wsx, stream=stream.cuda_stream),
                                   args.energy_seconds)
                if r is None:
                    d = None
                    break
                d[v] = r
            if d is None:
                energy = None
                break
            energy[j.kernel] = d

    # ---- the oracle on this host: the full config, all cores; and one thread at <= 2^24 units
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        rate, secs, cores, desc = oracle_rate(jobs, 1.0)
        frac1 = min(1.0, min((1 << 24) / j.n for j in jobs))
        rate1, secs1, _, desc1 = oracle_rate(jobs, frac1, threads=1)
        cpu = {"value": round(rate, 3) if rate else None, "unit": "GB/s", "cores": cores, "kind": "oracle",
               "sample": f"the full config, one run per kernel: {desc}", "seconds": round(secs, 2),
               "cpu": cpu_model(), "affinity_cores": len(os.sched_getaffinity(0)),
               "one_thread": {"value": round(rate1, 3) if rate1 else None, "unit": "GB/s", "cores": 1,
                              "sample": f"{frac1:.4g} of every kernel: {desc1}", "seconds": round(secs1, 2)}}

    if rank == 0:
        line = {
            "metric": METRIC, "value": round(value, 1) if value else None, "unit": "GB/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms_total / args.steps, 3),
            "higher_is_better": True, "scaling": scaling, "vs_baseline": None, "dtype": "u32/f32/u8x4",
            "data": "synthetic",
            "config": {"workload": workloads.CONFIG_TITLES[args.config], "preset": args.config,
                       "variants": variants, "l2": "every input > 126 MB L2 (no flush needed)",
                       "parallelism": f"dp{world} (data-sharded, {scaling})",
                       "value": "baseline (none) HBM GB/s: sum of algorithmic bytes / sum of none launch times"},
            "step_gbs_all_variants": round(step_bytes * args.steps * world / (ms_total * 1e-3) / 1e9, 1),
            "slowdown_geomean": slowdown_geomean, "baseline_frac": baseline_frac,
            "kernels": kernels, "rest10": rest or None, "graph_launch": graph_us, "roofline": roofline,
            "cpu_baseline": cpu, "e2e": e2e,
            "attribution": attribution, "extra_variants": extra, "energy": energy,
            "gpu_launches": counts["gpu_launches"], "err_count": errs,
            "clocks": clk.summary(),
        }
        print(json.dumps(line), flush=True)
    if peer_fwt is not None:
        peer_fwt.close()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
