"""Benchmark workloads: BASELINE.json configs as named presets.

A Job is one kernel at one size: host inputs (numpy, from the seeded
generators in inputs.py) or a device-side generator for the largest inputs,
device buffers in schema order, and the kernel's algorithmic HBM bytes per
launch (SURVEY 8(d) / DESIGN.md section 7).  No method arithmetic lives here.
Shards: rank r of G takes rows/elements [r*n, (r+1)*n) of the global index
space (weak scaling: fixed per-GPU size).

`bound` is the roofline class SURVEY 8(d) assigns (SURVEY.md:548-552): "hbm"
(streaming; the >= 70 % target applies), "latency" (BinarySearch: random
sectors), "mufu" (BlackScholes: MUFU ~ HBM), "l2" (FloydWarshall: the matrix
stays L2-resident), "tensor" (MatrixMultiplication), "alu" (BinomialOption).
"""
from __future__ import annotations

import dataclasses

import numpy as np
import torch

from . import inputs

MiB = 1 << 20


@dataclasses.dataclass
class Job:
    kernel: str
    n: int
    dims: tuple
    host_in: list          # numpy arrays, schema order, None for outputs
    out_shapes: list       # (index, nbytes) of output buffers
    alg_bytes: int         # algorithmic HBM bytes per launch
    unit: str              # what n counts
    bound: str = "hbm"
    note: str = ""
    dev: list | None = None
    dev_gen: object = None  # callable(i) -> device tensor of input i (instead of host_in[i])

    @property
    def mem_subset(self) -> bool:
        """The survey's memory-bound subset (SURVEY.md:548): R, T, Sobel, PS, FWT, DCT."""
        return self.kernel in ("reduction", "transpose", "sobel", "prefixsum", "fwt", "dct")

    def device_buffers(self):
        """Allocate device buffers once (inputs copied or generated in HBM, outputs zeroed)."""
        if self.dev is None:
            bufs = []
            for i, h in enumerate(self.host_in):
                if h is not None:
                    bufs.append(_to_dev(h))
                elif i not in dict(self.out_shapes):
                    bufs.append(self.dev_gen(i))
                else:
                    nbytes = dict(self.out_shapes)[i]
                    bufs.append(torch.zeros(max(nbytes // 4, 4), dtype=torch.int32, device="cuda")[: nbytes // 4])
            self.dev = bufs
        return self.dev

    @property
    def host_inputs(self) -> bool:
        return all(h is not None for i, h in enumerate(self.host_in) if i not in dict(self.out_shapes))

    def pinned_host(self):
        """Pinned host buffers (inputs filled, outputs empty) for the end-to-end call."""
        hb = []
        for i, h in enumerate(self.host_in):
            if h is not None:
                t = torch.from_numpy(_as_signed(h).reshape(-1).copy()).pin_memory()
            else:
                t = torch.empty(dict(self.out_shapes)[i] // 4, dtype=torch.int32).pin_memory()
            hb.append(t)
        return hb


def _as_signed(a: np.ndarray) -> np.ndarray:
    m = {np.dtype(np.uint32): np.int32, np.dtype(np.uint16): np.int16, np.dtype(np.uint8): np.uint8,
         np.dtype(np.uint64): np.int64}
    a = np.ascontiguousarray(a)
    return a.view(m.get(a.dtype, a.dtype))


def _to_dev(a: np.ndarray) -> torch.Tensor:
    a = _as_signed(a).reshape(-1)
    if a.dtype == np.uint8:
        a = a.view(np.int32)
    return torch.from_numpy(a.copy()).cuda()


# ---------------------------------------------------------------- per-kernel jobs

BINS_BYTES_PER_QUERY = 88  # 8 B (q, idx) + ~80 B of A no cache holds


def job_binarysearch(N, Q, seed=6, rank=0):
    A, _ = inputs.binarysearch_inputs(seed, N, 1)
    q = inputs.u32(seed, Q, rank * Q, stream=2)
    return Job("binarysearch", Q, (N, Q), [A, q, None], [(2, 4 * Q)], alg_bytes=BINS_BYTES_PER_QUERY * Q,
               unit="queries", bound="latency",
               note="88 B/query (SURVEY 8(d)): 8 B of q and idx + ~80 B of A per query -- the search levels that "
                    "are neither L2-resident (the top ~20 at N=2^26) nor inside the final shared sector (the last "
                    "3), i.e. 2-3 random 32-B sectors; below ncu's measured DRAM bytes per query")


def job_fwt(N, seed=5, rank=0):
    m = N.bit_length() - 1
    passes = 1 + (max(0, m - 12) + 6) // 7
    x = inputs.fwt_x(seed, N, rank * N)
    return Job("fwt", N, (), [x, None], [(1, 4 * N)], alg_bytes=8 * N * passes, unit="elements",
               note=f"{passes} passes x 8 B/elem")


def job_prefixsum(n, seed=4, rank=0):
    return Job("prefixsum", n, (), [inputs.prefixsum_x(seed, n, rank * n), None], [(1, 4 * n)],
               alg_bytes=8 * n, unit="elements")


def job_reduction(n, seed=2, rank=0):
    return Job("reduction", n, (), [inputs.reduction_x(seed, n, rank * n), None], [(1, 8)],
               alg_bytes=4 * n, unit="elements")


def job_transpose(H, W, seed=3, rank=0):
    A = inputs.transpose_a(seed, H, W, rank * H)
    return Job("transpose", H * W, (H, W), [A.view(np.uint32), None], [(1, 4 * H * W)],
               alg_bytes=8 * H * W, unit="elements")


def job_sobel(H, W, seed=7, rank=0, world=1):
    """Rank `rank` of `world` owns rows [rank H, (rank + 1) H) of a (world H)-row
    image; with world > 1 its input carries one halo row above / below
    (parallel.sobel_halo_rows), whose output rows are not part of the result."""
    r0 = rank * H
    lo, hi = (r0, r0 + H) if world == 1 else (max(0, r0 - 1), min(world * H, r0 + H + 1))
    I = inputs.sobel_image(seed, hi - lo, W, lo).view(np.uint32).reshape(-1)
    return Job("sobel", (hi - lo) * W, (hi - lo, W), [I, None], [(1, 4 * (hi - lo) * W)], alg_bytes=8 * H * W,
               unit="pixels", note="" if world == 1 else f"rows [{r0}, {r0 + H}) + halo rows [{lo}, {hi})")


def job_blackscholes(n, seed=1, rank=0, device_gen=False, offset=None):
    off = rank * n if offset is None else offset
    if device_gen:  # 2^30 options: generated in HBM (inputs.blackscholes_r_t, the same bits)
        return Job("blackscholes", n, (0,), [None, None, None], [(1, 4 * n), (2, 4 * n)], alg_bytes=12 * n,
                   unit="options", bound="mufu",
                   dev_gen=lambda i: inputs.blackscholes_r_t(seed, n, off))
    return Job("blackscholes", n, (0,), [inputs.blackscholes_r(seed, n, off), None, None],
               [(1, 4 * n), (2, 4 * n)], alg_bytes=12 * n, unit="options", bound="mufu")


def job_matmul(M, N, K, seed=10, rank=0, device_gen=False, row_offset=None):
    note = f"{2 * M * N * K:.3e} flop"
    ro = rank * M if row_offset is None else row_offset
    if device_gen:
        gen = {0: lambda: inputs.matmul_bf16_normal_t(seed, M, K, stream=22, row_offset=ro),
               1: lambda: inputs.matmul_bf16_normal_t(seed, N, K, stream=24)}
        return Job("matmul", M * N, (M, N, K), [None, None, None], [(2, 4 * M * N)],
                   alg_bytes=2 * (M * K + N * K) + 4 * M * N, unit="C elements", bound="tensor", note=note,
                   dev_gen=lambda i: gen[i]())
    A = inputs.matmul_bf16_normal(seed, M, K, stream=22, row_offset=ro)
    Bt = inputs.matmul_bf16_normal(seed, N, K, stream=24)
    return Job("matmul", M * N, (M, N, K), [A, Bt, None], [(2, 4 * M * N)],
               alg_bytes=2 * (M * K + N * K) + 4 * M * N, unit="C elements", bound="tensor", note=note)


def job_dct(H, W, seed=9, rank=0):
    return Job("dct", H * W, (H, W), [inputs.dct_x(seed, H, W, rank * H), None], [(1, 4 * H * W)],
               alg_bytes=8 * H * W, unit="elements")


def job_floydwarshall(n, seed=8):
    return Job("floydwarshall", n, (), [inputs.floydwarshall_w(seed, n), None], [(1, 4 * n * n)],
               alg_bytes=(n + 1) * 4 * n * n, unit="nodes", bound="l2",
               note="per pass: 4 B/elem read of D (L2-resident) + conditional writes; n passes + init")


def job_dwthaar1d(N, seed=11, rank=0):
    return Job("dwthaar1d", N, (), [inputs.dwt_x(seed, N, rank * N), None], [(1, 4 * N)],
               alg_bytes=8 * N, unit="samples", note="read x once, write y once (+N/256 B of approximations)")


def bitonic_launches(N):
    n = max(0, N.bit_length() - 1)
    return 1 + sum(-(-(s - 11) // 7) + 1 for s in range(12, n))


def job_bitonicsort(N, seed=21, rank=0):
    L = bitonic_launches(N)
    return Job("bitonicsort", N, (), [inputs.bitonic_keys(seed, N, rank * N), None], [(1, 4 * N)],
               alg_bytes=8 * N * L, unit="keys", note=f"{L} tile launches x 8 B/key (bitonic network, "
                                                      f"{(N.bit_length() - 1) * N.bit_length() // 2} passes)")


def job_binomialoption(n, seed=12, rank=0):
    return Job("binomialoption", n, (), [inputs.binomial_r(seed, n, rank * n), None], [(1, 4 * n)],
               alg_bytes=8 * n, unit="options", bound="alu",
               note="254-step CRR lattice in registers: ~64.8k flop/option (2 flop/node/step); HBM 8 B/option")


# ---------------------------------------------------------------- BASELINE.json configs

STRONG_CONFIGS = ("bs30", "mm16k")  # BASELINE.json configs[4]: a fixed global problem split over the GPUs


def _bs_strong(n_total, rank, world):
    off, cnt = strong_range(n_total, world, rank, 4)
    return job_blackscholes(cnt, rank=rank, device_gen=True, offset=off)


def _mm_strong(M, N, K, rank, world):
    off, cnt = strong_range(M, world, rank, 128)
    return job_matmul(cnt, N, K, rank=rank, device_gen=True, row_offset=off)


def strong_range(n_total: int, world: int, rank: int, align: int = 1):
    units = n_total // align
    lo, hi = units * rank // world, units * (rank + 1) // world
    return lo * align, (hi - lo) * align


def config_jobs(name: str, rank: int = 0, world: int = 1):
    if ":" in name:          # "<config>:<kernel>[,<kernel>]" -- a subset of a config (quick timing)
        base, ks = name.split(":", 1)
        keep = set(ks.split(","))
        return [j for j in config_jobs(base, rank, world) if j.kernel in keep]
    if name == "suite":      # configs[1]: the APP SDK-style suite, "paper's sizes"; weak scaling
        return [job_binarysearch(1 << 26, 1 << 24, rank=rank), job_fwt(1 << 26, rank=rank),
                job_prefixsum(1 << 26, rank=rank), job_reduction(1 << 26, rank=rank),
                job_transpose(8192, 8192, rank=rank), job_sobel(8192, 8192, rank=rank, world=world)]
    if name == "suite28":    # configs[2]: 2^28 elements
        return [job_binarysearch(1 << 28, 1 << 26, rank=rank), job_fwt(1 << 28, rank=rank),
                job_prefixsum(1 << 28, rank=rank), job_reduction(1 << 28, rank=rank),
                job_transpose(16384, 16384, rank=rank), job_sobel(16384, 16384, rank=rank, world=world)]
    if name == "bs16":       # configs[0]
        return [job_blackscholes(1 << 16, rank=rank)]
    if name == "bs30":       # configs[4] (BlackScholes part): 2^30 options split over the GPUs (strong)
        return [_bs_strong(1 << 30, rank, world)]
    if name == "mm16k":      # configs[4] (MatrixMultiplication part): rows of 16384^3 split (strong)
        return [_mm_strong(16384, 16384, 16384, rank, world)]
    if name == "rest10":     # the four BASELINE.json kernels outside configs[1] (bench.py's all-10 geomean)
        return [_bs_strong(1 << 30, rank, world), job_floydwarshall(4096),
                job_dct(8192, 8192, rank=rank), _mm_strong(16384, 16384, 16384, rank, world)]
    if name == "mm8k":
        return [job_matmul(8192, 8192, 8192, rank=rank)]
    if name == "fwdct":      # configs[3]
        return [job_floydwarshall(4096), job_dct(8192, 8192, rank=rank)]
    if name == "comm":       # the paper's communication-stress kernels
        return [job_dwthaar1d(1 << 26, rank=rank), job_bitonicsort(1 << 26, rank=rank),
                job_binomialoption(1 << 17, rank=rank)]
    if name == "small":      # smoke-sized
        return [job_binarysearch(1 << 16, 1 << 14, rank=rank), job_fwt(1 << 14, rank=rank),
                job_prefixsum(1 << 16, rank=rank), job_reduction(1 << 16, rank=rank),
                job_transpose(256, 256, rank=rank), job_sobel(256, 256, rank=rank)]
    raise ValueError(f"unknown config {name}")


CONFIG_TITLES = {
    "suite": "APP SDK-style suite (BinarySearch N=2^26 Q=2^24, FWT 2^26, PrefixSum 2^26, Reduction 2^26, "
             "Transpose 8192^2, Sobel 8192^2) x {none, intra_smem, intra_reg, inter_group}",
    "suite28": "suite at 2^28 elements (BinarySearch N=2^28 Q=2^26, Transpose/Sobel 16384^2)",
    "bs16": "BlackScholes 2^16 options",
    "bs30": "BlackScholes 2^30 options",
    "rest10": "BlackScholes 2^30, FloydWarshall 4096, DCT 8192^2, MatrixMultiplication 16384^3",
    "small": "suite at smoke sizes",
    "mm16k": "MatrixMultiplication 16384^3 bf16 -> fp32 (tcgen05)",
    "mm8k": "MatrixMultiplication 8192^3 bf16 -> fp32 (tcgen05)",
    "fwdct": "FloydWarshall 4096 nodes + DCT 8192^2",
    "comm": "communication-stress kernels (SURVEY 8(f) rank 2): DwtHaar1D 2^26, BitonicSort 2^26, "
            "BinomialOption 2^17 options",
}
