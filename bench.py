#!/usr/bin/env python
"""bench.py -- RMT slowdown per variant and baseline HBM GB/s vs peak
(BASELINE.json metric) on the APP SDK-style suite (BASELINE.json configs[1]).

One step = one pass of the whole hot path over one batch of synthetic input:
every kernel of the config launched once under each variant
(none, intra_smem, intra_reg, inter_group) through the C ABI (librmt.so).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config suite] [--impl rmt|reference]

value   = whole-job algorithmic HBM bytes of all launches / max-over-ranks device time
          (GB/s; inputs resident in HBM; every input > L2, so no flush is needed).
e2e     = the same metric through rmt_run_host (host pinned buffers; H2D of each
          launch's inputs and D2H of its outputs inside the timed region).
slowdown= per kernel t(variant)/t(none) and the geomean per variant.
The reference arm (--impl reference) is the CPU oracle (oracle/), timed as it
stands on this host's cores on a bounded sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import math
import os
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
    p.add_argument("--variants", default=",".join(VARIANTS))
    p.add_argument("--extra-variants", default=",".join(EXTRA_VARIANTS),
                   help="variants timed per launch after the timed region (reported, not in the step)")
    p.add_argument("--energy-seconds", type=float, default=0.5,
                   help="per (kernel, variant) NVML energy window; 0 disables the energy table")
    p.add_argument("--ablations", action="store_true",
                   help="also time the INFLATE and NOCOMM ablations per kernel x RMT variant (cost attribution)")
    p.add_argument("--dist-backend", default="nccl",
                   help="nccl (one GPU per rank); gloo only to exercise the multi-rank path on one GPU")
    return p.parse_args()


def load_peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(path) as f:
            pk = json.load(f)
        return float(pk["hbm_gbs"]), "measured (MEASURED_PEAKS.json)"
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
def oracle_sample_rate(jobs, min_seconds=1.0):
    """Time the oracle as it stands on a bounded sample of every job; return
    (equivalent GB/s, seconds, cores, description).  Rates are converted to the
    GPU metric with each job's full-size algorithmic bytes per unit."""
    import numpy as np

    import oracle
    from paper_conf_isca_waddenlgss14_b200 import inputs

    total_bytes_equiv = 0.0
    total_s = 0.0
    desc = []
    for j in jobs:
        bpu = j.alg_bytes / j.n
        if j.kernel == "binarysearch":
            A = j.host_in[0]
            q = inputs.u32(6, 1 << 20, 0, stream=2)
            fn, units, what = (lambda: oracle.binarysearch(A, q)), q.size, f"Q=2^20 on N={A.size}"
        elif j.kernel == "fwt":
            x = j.host_in[0][: 1 << 22]
            fn, units, what = (lambda: oracle.fwt_f64(x)), x.size, "N=2^22"
        elif j.kernel == "prefixsum":
            x = j.host_in[0][: 1 << 24]
            fn, units, what = (lambda: oracle.prefixsum_u32(x)), x.size, "n=2^24"
        elif j.kernel == "reduction":
            x = j.host_in[0][: 1 << 24]
            fn, units, what = (lambda: oracle.reduction_u32(x)), x.size, "n=2^24"
        elif j.kernel == "transpose":
            H, W = j.dims
            h = max(4, min(H, (1 << 24) // W))
            A = np.ascontiguousarray(j.host_in[0].reshape(H, W)[:h])
            fn, units, what = (lambda: oracle.transpose_u32(A)), A.size, f"{h}x{W}"
        elif j.kernel == "sobel":
            H, W = j.dims
            h = max(3, min(H, (1 << 23) // W))
            I = np.ascontiguousarray(j.host_in[0].reshape(H, W)[:h]).view(np.uint8).reshape(h, W, 4)
            fn, units, what = (lambda: oracle.sobel(I)), h * W, f"{h}x{W}"
        elif j.kernel == "blackscholes":
            r = j.host_in[0][: 1 << 22]
            fn, units, what = (lambda: oracle.blackscholes(r)), r.size, f"n={r.size}"
        elif j.kernel == "dwthaar1d":
            x = j.host_in[0][: 1 << 22]
            fn, units, what = (lambda: oracle.dwthaar1d_f64(x)), x.size, "N=2^22"
        elif j.kernel == "bitonicsort":
            k = j.host_in[0][: 1 << 22]
            fn, units, what = (lambda: oracle.sort_u32(k)), k.size, "N=2^22"
        elif j.kernel == "binomialoption":
            r = j.host_in[0][: 1 << 12]
            fn, units, what = (lambda: oracle.binomialoption(r)), r.size, "n=2^12"
        elif j.kernel == "matmul":
            # full-K dot products for a 128 x 128 block of C (units = C elements)
            A, Bt = j.host_in[0], j.host_in[1]
            M, N, K = j.dims
            As = np.ascontiguousarray(A.reshape(M, K)[:128])
            Bs = np.ascontiguousarray(Bt.reshape(N, K)[:128])
            fn, units, what = (lambda: oracle.matmul_bf16(As, Bs)), 128 * 128, f"C[0:128,0:128] at K={K}"
        elif j.kernel == "floydwarshall":
            # the n'^3 relaxations of an n' = 512 sub-problem, converted to the
            # full problem's units (n^3 relaxations per n nodes)
            n = j.n
            m = min(n, 512)
            Wm = np.ascontiguousarray(j.host_in[0].reshape(n, n)[:m, :m])
            fn, units, what = (lambda: oracle.floydwarshall(Wm)), m ** 3 / n ** 2, f"n'={m} sub-graph"
        elif j.kernel == "dct":
            H, W = j.dims
            h = max(8, min(H, (1 << 22) // W) // 8 * 8)
            X = np.ascontiguousarray(j.host_in[0].reshape(H, W)[:h])
            fn, units, what = (lambda: oracle.dct8x8(X)), h * W, f"{h}x{W}"
        else:
            continue
        reps, t0 = 0, time.perf_counter()
        while True:
            fn()
            reps += 1
            dt = time.perf_counter() - t0
            if dt >= min_seconds:
                break
        total_bytes_equiv += reps * units * bpu
        total_s += dt
        desc.append(f"{j.kernel} {what} x{reps}")
    return total_bytes_equiv / total_s / 1e9, total_s, oracle.num_threads(), "; ".join(desc)


# ---------------------------------------------------------------- main
def main():
    args = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))

    from paper_conf_isca_waddenlgss14_b200 import workloads

    if args.impl == "reference":
        if rank != 0:
            return  # rank 0 alone runs the CPU reference arm
        jobs = workloads.config_jobs(args.config, 0)
        for _ in range(args.warmup):
            pass
        times = []
        rate = None
        for _ in range(args.steps):
            rate, secs, cores, desc = oracle_sample_rate(jobs, min_seconds=0.5)
            times.append(secs)
        line = {
            "impl": "reference", "metric": METRIC, "value": round(rate, 3), "unit": "GB/s",
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": round(1e3 * statistics.mean(times), 3), "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "u32/f32", "data": "synthetic",
            "config": {"workload": workloads.CONFIG_TITLES[args.config], "preset": args.config},
            "cpu_baseline": {"value": round(rate, 3), "unit": "GB/s", "cores": cores, "kind": "oracle",
                             "sample": desc},
            "e2e": {"value": round(rate, 3), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
        }
        print(json.dumps(line), flush=True)
        return

    import torch
    import torch.distributed as dist

    from paper_conf_isca_waddenlgss14_b200 import rmt

    dev_index = local_rank % max(1, torch.cuda.device_count())
    torch.cuda.set_device(dev_index)
    if world > 1:
        if args.dist_backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", dev_index))
        else:
            dist.init_process_group(args.dist_backend)
    variants = [v for v in args.variants.split(",") if v]
    jobs = workloads.config_jobs(args.config, rank)
    stream = torch.cuda.current_stream()
    err = torch.zeros(1, dtype=torch.int64, device="cuda")
    ws = {}
    ws_red = {}
    for j in jobs:
        j.device_buffers()
        for v in variants:
            ws[(j.kernel, v)] = rmt.make_workspace(j.kernel, v, j.n, j.dims)
            if j.kernel == "prefixsum":
                ws_red[v] = rmt.make_workspace("reduction", v, j.n)
    torch.cuda.synchronize()

    launches = [(j, v) for j in jobs for v in variants]
    ev = {(j.kernel, v): [] for j, v in launches}
    counts = {"gpu_launches": 0}

    from paper_conf_isca_waddenlgss14_b200 import parallel
    s_tmp = torch.zeros(2, dtype=torch.int32, device="cuda")

    def one(j, v):
        """One launch of job j under variant v; for N > 1 the kernels that need a
        cross-shard exchange do it here."""
        if world > 1 and j.kernel == "prefixsum":
            # local total (Reduction kernel) -> all-gather -> carry-in -> scan
            parallel.global_prefixsum(j.dev[0], j.dev[1], s_tmp, err, rmt, variant=v,
                                      ws_red=ws_red[v], ws_ps=ws[(j.kernel, v)])
            return 2
        nk = rmt.launch(j.kernel, v, j.dev, j.n, err, dims=j.dims, workspace=ws[(j.kernel, v)],
                        stream=stream.cuda_stream)
        if world > 1 and j.kernel == "reduction":
            parallel.allreduce_sum_(j.dev[1].view(torch.int64))
        return nk

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
        if world > 1:
            parallel.allreduce_sum_(err)  # error counters of every rank

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
    if world > 1:
        tt = torch.tensor([ms_total], dtype=torch.float64, device="cuda")
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        ms_total = float(tt.item())
    errs = int(err.item())

    # per-launch device times
    per = {}
    for (k, v), lst in ev.items():
        per[(k, v)] = statistics.median(a.elapsed_time(b) for a, b in lst)
    peak, peak_src = load_peaks()
    step_bytes = sum(j.alg_bytes for j, _ in launches)
    value = step_bytes * args.steps * world / (ms_total * 1e-3) / 1e9

    kernels = {}
    slow = {v: [] for v in variants if v != "none"}
    for j in jobs:
        d = {}
        for v in variants:
            ms = per[(j.kernel, v)]
            gbs = j.alg_bytes / (ms * 1e-3) / 1e9
            d[v] = {"ms": round(ms, 4), "gbs": round(gbs, 1), "frac": round(gbs / peak, 4)}
            if job_flops(j):
                tf = job_flops(j) / (ms * 1e-3) / 1e12
                d[v]["tflops"] = round(tf, 1)
                d[v]["tensor_frac"] = round(tf / load_tensor_peak()[0], 4)
            if v != "none" and "none" in variants:
                sd = ms / per[(j.kernel, "none")]
                d[v]["slowdown"] = round(sd, 3)
                slow[v].append(sd)
        d["bound"] = j.bound
        kernels[j.kernel] = d
    geo = {v: round(math.exp(sum(math.log(x) for x in s) / len(s)), 3) for v, s in slow.items() if s}
    geo_mem = {}
    for v, s in slow.items():
        mem = [per[(j.kernel, v)] / per[(j.kernel, "none")] for j in jobs if j.bound == "hbm"]
        if mem:
            geo_mem[v] = round(math.exp(sum(math.log(x) for x in mem) / len(mem)), 3)

    # dominant kernel (largest share of the step) -> roofline
    dom = max(launches, key=lambda jv: per[(jv[0].kernel, jv[1])])
    dj, dv = dom
    dms = per[(dj.kernel, dv)]
    ach = dj.alg_bytes / (dms * 1e-3) / 1e9
    traffic = load_traffic().get(f"{dj.kernel}/{dv}")
    roofline = {"bound": "hbm", "achieved": round(ach, 1), "peak": peak, "unit": "GB/s",
                "frac": round(ach / peak, 4), "traffic": traffic, "kernel": f"{dj.kernel}/{dv}",
                "share_of_step": round(dms / (ms_total / args.steps), 3), "peak_source": peak_src,
                "algorithmic_bytes_per_launch": dj.alg_bytes}
    if dj.bound == "tensor" and job_flops(dj):
        tpk, tsrc = load_tensor_peak()
        tach = job_flops(dj) / (dms * 1e-3) / 1e12
        roofline.update({"bound": "tensor", "achieved": round(tach, 1), "peak": tpk, "unit": "TFLOP/s",
                         "frac": round(tach / tpk, 4), "peak_source": tsrc,
                         "algorithmic_flops_per_launch": job_flops(dj),
                         "note": "both replicas run the full contraction on the tensor pipe; achieved counts "
                                 "the algorithmic 2MNK once"})
    best_none = max((j for j in jobs if j.bound == "hbm"), key=lambda j: j.alg_bytes / per[(j.kernel, "none")],
                    default=None)

    # end-to-end through the public C ABI with host buffers
    e2e = None
    if args.e2e_steps > 0:
        hosts = {j.kernel: j.pinned_host() for j in jobs}
        h2d = d2h = 0
        for j, v in launches:  # warm
            rmt.run_host(j.kernel, v, hosts[j.kernel], j.dev, j.n, err, dims=j.dims, workspace=ws[(j.kernel, v)])
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(args.e2e_steps):
            for j, v in launches:
                _, hb, db = rmt.run_host(j.kernel, v, hosts[j.kernel], j.dev, j.n, err, dims=j.dims,
                                         workspace=ws[(j.kernel, v)])
                h2d += hb
                d2h += db
        e1.record(stream)
        torch.cuda.synchronize()
        ems = e0.elapsed_time(e1)
        if world > 1:
            tt = torch.tensor([ems], dtype=torch.float64, device="cuda")
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
            ems = float(tt.item())
        e2e = {"value": round(step_bytes * args.e2e_steps * world / (ems * 1e-3) / 1e9, 3), "unit": "GB/s",
               "h2d_bytes_per_step": h2d // args.e2e_steps, "d2h_bytes_per_step": d2h // args.e2e_steps,
               "ms_per_step": round(ems / args.e2e_steps, 3)}

    # Cost attribution "as the paper does": t(none) ->
    # inflate (none with the RMT variant's per-SM residency: redundant scheduling)
    # -> nocomm (both replicas, no exchange: redundant compute) -> full (+ comm).
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

    # B200-native extension variants: per-launch medians outside the timed step
    extra = None
    xvars = [v for v in args.extra_variants.split(",") if v and v not in variants]
    if xvars and "none" in variants:
        extra = {"kernels": {}, "slowdown_geomean": {}}
        xs = {v: [] for v in xvars}
        err.zero_()
        for j in jobs:
            d = {}
            for v in xvars:
                wsx = rmt.make_workspace(j.kernel, v, j.n, j.dims)
                ts = []
                for r in range(5):
                    a = torch.cuda.Event(enable_timing=True)
                    b = torch.cuda.Event(enable_timing=True)
                    a.record(stream)
                    rmt.launch(j.kernel, v, j.dev, j.n, err, dims=j.dims, workspace=wsx, stream=stream.cuda_stream)
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
        extra["slowdown_geomean"] = {v: round(math.exp(sum(math.log(x) for x in s_) / len(s_)), 3)
                                     for v, s_ in xs.items()}
        extra["err_count"] = int(err.item())

    # average power and energy per launch for every kernel x variant
    energy = None
    if args.energy_seconds > 0 and world == 1:
        energy = {}
        allv = variants + [v for v in args.extra_variants.split(",") if v and v not in variants]
        for j in jobs:
            d = {}
            for v in allv:
                wsx = ws.get((j.kernel, v))
                if wsx is None:
                    wsx = rmt.make_workspace(j.kernel, v, j.n, j.dims)
                r = measure_energy(dev_index, lambda: rmt.launch(j.kernel, v, j.dev, j.n, err, dims=j.dims,
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
        err.zero_()

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        rate, secs, cores, desc = oracle_sample_rate(jobs)
        cpu = {"value": round(rate, 3), "unit": "GB/s", "cores": cores, "kind": "oracle", "sample": desc,
               "seconds": round(secs, 2)}

    if rank == 0:
        line = {
            "metric": METRIC, "value": round(value, 1), "unit": "GB/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(ms_total / args.steps, 3), "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "u32/f32/u8x4", "data": "synthetic",
            "config": {"workload": workloads.CONFIG_TITLES[args.config], "preset": args.config,
                       "variants": variants, "l2": "every input > 126 MB L2 (no flush needed)",
                       "parallelism": f"dp{world} (data-sharded, weak)"},
            "slowdown_geomean": geo, "slowdown_geomean_hbm_kernels": geo_mem,
            "baseline_best": ({"kernel": best_none.kernel,
                               "gbs": kernels[best_none.kernel]["none"]["gbs"],
                               "frac": kernels[best_none.kernel]["none"]["frac"]} if best_none else None),
            "kernels": kernels, "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e,
            "attribution": attribution, "extra_variants": extra, "energy": energy,
            "gpu_launches": counts["gpu_launches"], "err_count": errs,
            "clocks": clk.summary(),
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
