"""Seeded, counter-based synthetic input generators.

This module is shared by the CUDA path's tests/bench AND by the oracle side
(DESIGN.md "Input recipe").  It deliberately holds none of the method's
arithmetic: no RMT, no kernel definitions -- only "element i of stream `seed`"
= splitmix64(seed, i), mapped to the value distributions of the paper's
workloads (AMD APP SDK-style random inputs, "input sizes were
scaled to the maximum size ...").  Because every value is a pure function of
(seed, global index), a shard [off, off+n) on any rank reproduces exactly the
same numbers as the corresponding slice of the 1-GPU input.

All functions return numpy arrays on the host; callers copy them to the GPU.
"""
from __future__ import annotations

import numpy as np

_GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)
_CHUNK = 1 << 24


def _mix(z: np.ndarray) -> np.ndarray:
    z = (z ^ (z >> np.uint64(30))) * _M1
    z = (z ^ (z >> np.uint64(27))) * _M2
    return z ^ (z >> np.uint64(31))


def u64(seed: int, n: int, offset: int = 0, stream: int = 0) -> np.ndarray:
    """uint64 stream: splitmix64 of (seed, stream) keyed counter, element offset+i."""
    key = _mix(np.array([(seed * 0x100000001B3 + stream * 0x1000193 + 1) & (2**64 - 1)],
                        dtype=np.uint64))[0]
    out = np.empty(n, dtype=np.uint64)
    with np.errstate(over="ignore"):
        for s in range(0, n, _CHUNK):
            e = min(n, s + _CHUNK)
            idx = np.arange(offset + s, offset + e, dtype=np.uint64)
            out[s:e] = _mix(idx * _GOLDEN + key)
    return out


def u32(seed: int, n: int, offset: int = 0, stream: int = 0) -> np.ndarray:
    return (u64(seed, n, offset, stream) >> np.uint64(32)).astype(np.uint32)


def uniform_f32(seed: int, n: int, offset: int = 0, stream: int = 0) -> np.ndarray:
    """U[0,1) with 24 random bits: every value k*2^-24 is exact in fp32."""
    k = (u64(seed, n, offset, stream) >> np.uint64(40)).astype(np.float64)
    return (k * (2.0 ** -24)).astype(np.float32)


# --------------------------------------------------------------------------
# Per-workload recipes (SURVEY.md 8(d) synthetic inputs)
# --------------------------------------------------------------------------

def blackscholes_r(seed: int, n: int, offset: int = 0) -> np.ndarray:
    """One U[0,1) draw per option (APP-SDK style; the kernel maps r -> S,K,T,R,sigma)."""
    return uniform_f32(seed, n, offset)


def blackscholes_indep(seed: int, n: int, offset: int = 0) -> np.ndarray:
    """Independent parameters (SURVEY 8(c) "bs_indep"): uniform S in [5,30],
    K in [1,100], T in [0.25,10], R in [0.01,0.05], sigma in [0.1,0.5]; returned
    as float32 planes (5, n): S | K | T | R | sigma (the ABI's mode-1 layout)."""
    lo = (5.0, 1.0, 0.25, 0.01, 0.10)
    hi = (30.0, 100.0, 10.0, 0.05, 0.50)
    out = np.empty((5, n), np.float32)
    for k in range(5):
        u = uniform_f32(seed, n, offset, stream=30 + k).astype(np.float64)
        out[k] = (lo[k] + (hi[k] - lo[k]) * u).astype(np.float32)
    return out


# Hand-picked option rows (S, K, T, R, sigma) for the independent-parameter
# mode: textbook points, at/in/out of the money, negative d1 and d2, extremes
# of the bs_indep ranges.
BS_EDGE_ROWS = [
    (100.0, 100.0, 1.0, 0.05, 0.20),   # textbook ATM point (C = 10.45058, P = 5.57353)
    (42.0, 40.0, 0.5, 0.10, 0.20),     # Hull, Options Futures & Other Derivatives, Ex. 15.6 (C ~ 4.76, P ~ 0.81)
    (30.0, 1.0, 10.0, 0.05, 0.50),     # deep in the money call
    (5.0, 100.0, 0.25, 0.01, 0.10),    # deep out of the money call (d1 ~ -60)
    (20.0, 40.0, 2.0, 0.03, 0.30),     # d1 < 0, d2 < 0
    (25.0, 30.0, 5.0, 0.02, 0.15),     # slightly out of the money: d1, d2 just below 0
    (10.0, 10.5, 0.25, 0.01, 0.50),    # near the money, short expiry, high vol
    (5.0, 1.0, 0.25, 0.05, 0.10),      # deep ITM, short expiry
    (30.0, 100.0, 10.0, 0.01, 0.50),   # OTM, long expiry, high vol
    (12.0, 11.0, 0.25, 0.05, 0.10),    # d1 > 0, d2 > 0
    (7.5, 8.0, 3.0, 0.04, 0.40),       # d1 > 0 > d2
    (1.0, 100.0, 10.0, 0.05, 0.10),    # extreme OTM: prices underflow to 0
]


def blackscholes_edges() -> np.ndarray:
    """BS_EDGE_ROWS as float32 planes (5, n), n padded to a multiple of 4 by
    repeating the first row."""
    rows = list(BS_EDGE_ROWS)
    while len(rows) % 4:
        rows.append(rows[0])
    return np.ascontiguousarray(np.array(rows, dtype=np.float32).T)


def with_specials(x: np.ndarray, seed: int, frac: float = 0.01, kinds=("nan", "+0", "-0")) -> np.ndarray:
    """A copy of float32 x with a seeded fraction of entries replaced by IEEE
    special values (quiet NaN, +0, -0, optionally +/-inf): the bitwise-compare
    reading R-RMT4 must give no false alarm on any of them."""
    x = np.array(x, dtype=np.float32, copy=True)
    flat = x.reshape(-1)
    n = flat.size
    m = max(1, int(n * frac))
    pos = (u64(seed, m, 0, stream=40) % np.uint64(max(n, 1))).astype(np.int64)
    sel = (u32(seed, m, 0, stream=41) % np.uint32(len(kinds))).astype(np.int64)
    vals = {"nan": np.float32(np.nan), "+0": np.float32(0.0), "-0": np.float32(-0.0),
            "+inf": np.float32(np.inf), "-inf": np.float32(-np.inf)}
    for i, k in enumerate(kinds):
        flat[pos[sel == i]] = vals[k]
    return x


def binarysearch_inputs(seed: int, N: int, Q: int, q_offset: int = 0):
    """Sorted, strictly increasing u32 A[N] spread over the full u32 range, and
    uniform u32 queries q[Q].  A[i] = i*stride + (h(i) mod stride) (no prefix sum
    needed to make it sorted)."""
    stride = (1 << 32) // N
    if stride < 1:
        raise ValueError("N too large for u32 keys")
    h = u32(seed, N, 0, stream=1).astype(np.uint64)
    A = (np.arange(N, dtype=np.uint64) * np.uint64(stride) + h % np.uint64(stride)).astype(np.uint32)
    q = u32(seed, Q, q_offset, stream=2)
    return A, q


def binarysearch_dups(seed: int, N: int, Q: int, distinct: int = 1000):
    """Sorted A[N] with heavy duplication: values from a pool of `distinct`
    random keys plus 0 and 0xFFFFFFFF (both extremes present, in runs);
    queries drawn from the pool, its neighbours (key - 1, key + 1) and the two
    extremes, so every lower_bound lands on the first element of a run."""
    pool = np.unique(np.concatenate([u32(seed, distinct, 0, stream=42),
                                     np.array([0, 1, 0xFFFFFFFE, 0xFFFFFFFF], np.uint32)]))
    A = np.sort(pool[(u32(seed, N, 0, stream=43) % np.uint32(pool.size)).astype(np.int64)])
    pick = pool[(u32(seed, Q, 0, stream=44) % np.uint32(pool.size)).astype(np.int64)].astype(np.int64)
    delta = (u32(seed, Q, 0, stream=45) % np.uint32(3)).astype(np.int64) - 1
    q = np.clip(pick + delta, 0, 0xFFFFFFFF).astype(np.uint32)
    q[: min(Q, 4)] = np.array([0, 0xFFFFFFFF, 1, 0xFFFFFFFE], np.uint32)[: min(Q, 4)]
    return A.astype(np.uint32), q


def fwt_x(seed: int, n: int, offset: int = 0) -> np.ndarray:
    """U[-1,1) fp32 (exact: 2*k*2^-24 - 1)."""
    return (uniform_f32(seed, n, offset) * np.float32(2.0) - np.float32(1.0)).astype(np.float32)


def fwt_ternary(seed: int, n: int, offset: int = 0) -> np.ndarray:
    """x in {-1,0,1} (exact-integer pin input for the FWT)."""
    return ((u32(seed, n, offset, stream=3) % np.uint32(3)).astype(np.int64) - 1).astype(np.float32)


def prefixsum_x(seed: int, n: int, offset: int = 0) -> np.ndarray:
    """u32 U{0..255}."""
    return (u32(seed, n, offset, stream=4) & np.uint32(0xFF)).astype(np.uint32)


def prefixsum_f32(seed: int, n: int, offset: int = 0) -> np.ndarray:
    """fp32 PrefixSum input (SURVEY 8(d) configs[1]: "+f32 U[0,1)")."""
    return uniform_f32(seed + 1000, n, offset)


def reduction_x(seed: int, n: int, offset: int = 0) -> np.ndarray:
    """u32 U{0..2^16-1}."""
    return (u32(seed, n, offset, stream=5) & np.uint32(0xFFFF)).astype(np.uint32)


def transpose_a(seed: int, H: int, W: int, row_offset: int = 0) -> np.ndarray:
    """f32 U[0,1), H x W row-major."""
    return uniform_f32(seed, H * W, row_offset * W, stream=6).reshape(H, W)


def sobel_image(seed: int, H: int, W: int, row_offset: int = 0) -> np.ndarray:
    """uchar4 image (H, W, 4): 64x64 checker blocks (edges) + diagonal ramp + 4-bit noise."""
    y = np.arange(row_offset, row_offset + H, dtype=np.int64)[:, None, None]
    x = np.arange(W, dtype=np.int64)[None, :, None]
    c = np.arange(4, dtype=np.int64)[None, None, :]
    block = (((x // 64) + (y // 64)) % 2) * 96
    ramp = (x % 64) + (y % 64) + 8 * c
    noise = (u32(seed, H * W * 4, row_offset * W * 4, stream=7).astype(np.int64)
             & 15).reshape(H, W, 4)
    return np.minimum(block + ramp + noise, 255).astype(np.uint8)


def floydwarshall_w(seed: int, n: int) -> np.ndarray:
    """Complete digraph, u32 weights U{1..200}, zero diagonal."""
    w = (u32(seed, n * n, 0, stream=8) % np.uint32(200) + np.uint32(1)).reshape(n, n)
    np.fill_diagonal(w, 0)
    return w.astype(np.uint32)


FW_INF = 0x3FFFFFFF  # "no edge" weight of the sparse FloydWarshall graphs


def floydwarshall_sparse(seed: int, n: int, p_edge: float = 0.05) -> np.ndarray:
    """Sparse digraph: each off-diagonal edge present with probability p_edge
    (weight U{1..200}), absent edges FW_INF = 0x3FFFFFFF (2 * FW_INF < 2^32: the
    u32 relaxation sum cannot wrap), zero diagonal.  Small p_edge leaves some
    pairs unreachable (their distance stays >= FW_INF)."""
    w = (u32(seed, n * n, 0, stream=8) % np.uint32(200) + np.uint32(1)).reshape(n, n)
    present = (u32(seed, n * n, 0, stream=46).astype(np.float64) * 2.0 ** -32).reshape(n, n) < p_edge
    w = np.where(present, w, np.uint32(FW_INF)).astype(np.uint32)
    np.fill_diagonal(w, 0)
    return w


def dct_x(seed: int, H: int, W: int, row_offset: int = 0) -> np.ndarray:
    """f32 U[0,255)."""
    return (uniform_f32(seed, H * W, row_offset * W, stream=9) * np.float32(255.0)).reshape(H, W)


def f32_to_bf16_bits(x: np.ndarray) -> np.ndarray:
    """Round-to-nearest-even fp32 -> bf16, returned as uint16 bit patterns."""
    b = np.ascontiguousarray(x, dtype=np.float32).view(np.uint32).astype(np.uint64)
    b = b + np.uint64(0x7FFF) + ((b >> np.uint64(16)) & np.uint64(1))
    return (b >> np.uint64(16)).astype(np.uint16)


def bf16_bits_to_f32(b: np.ndarray) -> np.ndarray:
    return (b.astype(np.uint32) << np.uint32(16)).view(np.float32)


def matmul_bf16_normal(seed: int, rows: int, cols: int, stream: int, row_offset: int = 0) -> np.ndarray:
    """bf16 N(0,1) (Box-Muller on two counter streams), returned as uint16 bits."""
    n = rows * cols
    off = row_offset * cols
    out = np.empty(n, np.uint16)
    for s in range(0, n, _CHUNK):
        e = min(n, s + _CHUNK)
        u1 = (u64(seed, e - s, off + s, stream=stream) >> np.uint64(11)).astype(np.float64) * 2.0 ** -53
        u2 = (u64(seed, e - s, off + s, stream=stream + 1) >> np.uint64(11)).astype(np.float64) * 2.0 ** -53
        g = np.sqrt(-2.0 * np.log1p(-u1)) * np.cos(2.0 * np.pi * u2)
        out[s:e] = f32_to_bf16_bits(g.astype(np.float32))
    return out.reshape(rows, cols)


def matmul_bf16_int(seed: int, rows: int, cols: int, stream: int, lo: int = -4, hi: int = 4,
                    row_offset: int = 0) -> np.ndarray:
    """Integer-valued bf16 in [lo, hi] (exactness pin input), uint16 bits."""
    n = rows * cols
    v = (u32(seed, n, row_offset * cols, stream=stream) % np.uint32(hi - lo + 1)).astype(np.int64) + lo
    return f32_to_bf16_bits(v.astype(np.float32)).reshape(rows, cols)


# ---- SURVEY 8(f) rank 2 kernels ----

def bitonic_keys(seed: int, n: int, offset: int = 0, bits: int = 32) -> np.ndarray:
    """u32 keys, uniform over [0, 2^bits) (bits < 32: duplicate-heavy)."""
    k = u32(seed, n, offset, stream=10)
    if bits < 32:
        k &= np.uint32((1 << bits) - 1)
    return k


def dwt_x(seed: int, n: int, offset: int = 0) -> np.ndarray:
    """f32 U[-1,1) signal (exact: 2*k*2^-24 - 1)."""
    return (uniform_f32(seed, n, offset, stream=11) * np.float32(2.0) - np.float32(1.0)).astype(np.float32)


def binomial_r(seed: int, n: int, offset: int = 0) -> np.ndarray:
    """One U[0,1) draw per option (APP-SDK style; the kernel maps r -> S, K, T)."""
    return uniform_f32(seed, n, offset, stream=12)


# --------------------------------------------------------------------------
# Device-side twins of the generators above (torch tensor ops, no method
# arithmetic): the same splitmix64 counter stream, bit for bit, produced in HBM
# for the bench's largest inputs (BlackScholes 2^30 options, MatrixMultiplication
# 16384^2 operands) where host generation would take minutes.
# tests/test_inputs_cpu.py pins u64_t / uniform_f32_t against the numpy versions.
# --------------------------------------------------------------------------

def _srl(z, k: int):
    """Logical right shift of int64 tensors holding uint64 bit patterns."""
    import torch
    return (z >> k) & ((1 << (64 - k)) - 1)


def _mix_t(z):
    M1 = 0xBF58476D1CE4E5B9 - (1 << 64)  # the same constants as int64 bit patterns
    M2 = 0x94D049BB133111EB - (1 << 64)
    z = (z ^ _srl(z, 30)) * M1
    z = (z ^ _srl(z, 27)) * M2
    return z ^ _srl(z, 31)


def u64_t(seed: int, n: int, offset: int = 0, stream: int = 0, device="cuda"):
    """int64 tensor with the bit patterns of u64(seed, n, offset, stream)."""
    import torch
    key = int(_mix(np.array([(seed * 0x100000001B3 + stream * 0x1000193 + 1) & (2**64 - 1)], dtype=np.uint64))[0])
    key = key - (1 << 64) if key >= (1 << 63) else key
    gold = 0x9E3779B97F4A7C15 - (1 << 64)
    out = torch.empty(n, dtype=torch.int64, device=device)
    for s in range(0, n, _CHUNK):
        e = min(n, s + _CHUNK)
        idx = torch.arange(offset + s, offset + e, dtype=torch.int64, device=device)
        out[s:e] = _mix_t(idx * gold + key)
    return out


def uniform_f32_t(seed: int, n: int, offset: int = 0, stream: int = 0, device="cuda"):
    import torch
    out = torch.empty(n, dtype=torch.float32, device=device)
    for s in range(0, n, _CHUNK):
        e = min(n, s + _CHUNK)
        k = _srl(u64_t(seed, e - s, offset + s, stream, device), 40).to(torch.float64)
        out[s:e] = (k * (2.0 ** -24)).to(torch.float32)
    return out


def blackscholes_r_t(seed: int, n: int, offset: int = 0, device="cuda"):
    return uniform_f32_t(seed, n, offset, 0, device)


def matmul_bf16_normal_t(seed: int, rows: int, cols: int, stream: int, row_offset: int = 0, device="cuda"):
    """bf16 N(0,1) on the device (Box-Muller on the same two counter streams as
    matmul_bf16_normal; the device log/cos may round a rare value differently
    from numpy's), returned as an int16 tensor of bf16 bit patterns."""
    import torch
    n = rows * cols
    off = row_offset * cols
    out = torch.empty(n, dtype=torch.bfloat16, device=device)
    for s in range(0, n, _CHUNK):
        e = min(n, s + _CHUNK)
        u1 = _srl(u64_t(seed, e - s, off + s, stream, device), 11).to(torch.float64) * 2.0 ** -53
        u2 = _srl(u64_t(seed, e - s, off + s, stream + 1, device), 11).to(torch.float64) * 2.0 ** -53
        g = torch.sqrt(-2.0 * torch.log1p(-u1)) * torch.cos(2.0 * np.pi * u2)
        out[s:e] = g.to(torch.float32).to(torch.bfloat16)
    return out.view(torch.int16)
