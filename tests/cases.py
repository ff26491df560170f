"""Per-kernel GPU test cases: seeded inputs (paper_conf_isca_waddenlgss14_b200.inputs),
sentinel-filled outputs, and the oracle check for each kernel at a given size.

A Case knows how to build a fresh set of device buffers in schema order, and
how to compare the GPU outputs with the oracle (tolerances per DESIGN.md
"Parity rules").
"""
from __future__ import annotations

import functools

import numpy as np
import torch

import oracle
from paper_conf_isca_waddenlgss14_b200 import inputs
from helpers import dev, host, out_like


class Case:
    kernel: str
    n: int
    dims: tuple = ()
    tag: str = ""  # input-set qualifier for test ids (specials, dups, sparse, ...)

    @property
    def id(self):
        return f"{self.kernel}-{self.n}{self.tag}"

    def buffers(self):
        """Fresh device buffers in schema order (outputs sentinel-filled)."""
        raise NotImplementedError

    def outputs(self, bufs):
        """Host copies of the output buffers (as comparable numpy arrays)."""
        raise NotImplementedError

    def check(self, outs):
        """Assert outputs match the oracle."""
        raise NotImplementedError

    def out_elems(self):
        """(buffer index, element count) of the first output buffer (STORE_* fault site)."""
        raise NotImplementedError

    def fault_target(self, rng):
        """(elem for rmt_inject_fault, word index in the first output buffer)."""
        b, ne = self.out_elems()
        e = int(rng.integers(0, ne))
        return e, e

    def fault_propagates(self):
        """True if a suppressed store feeds later computation (multi-pass, in place)."""
        return False

    def flipped_oracle(self, elem, bit):
        """Outputs the oracle predicts when input word `elem` (the kernel's LOAD
        fault site) has bit `bit` flipped -- an independent liveness prediction
        (SURVEY 8(c) C-FI); None where the site is not an input word or the
        oracle is not exact."""
        return None

    def commit_group(self, e):
        """Word indices of the first output buffer stored by the same commit as
        word e (one commit per store instruction; vector stores are 4 words)."""
        b, ne = self.out_elems()
        lo = e - e % 4
        return np.arange(lo, min(lo + 4, ne))


def _nan_aware_equal(got_bits, ref_bits):
    """Bitwise equality, except that any NaN matches any NaN (the CPU and the
    GPU quiet NaNs with different payloads; the RMT variants are still compared
    with `none` bit for bit)."""
    g = got_bits.view(np.float32)
    r = ref_bits.view(np.float32)
    gn, rn = np.isnan(g), np.isnan(r)
    return np.array_equal(gn, rn) and np.array_equal(got_bits[~gn], ref_bits[~rn])


def _flip(a, elem, bit):
    """Copy of array a with bit `bit` of 32-bit word `elem` flipped."""
    b = np.array(a, copy=True)
    w = b.reshape(-1).view(np.uint32)
    w[elem] ^= np.uint32(1 << bit)
    return b


class BlackScholes(Case):
    kernel = "blackscholes"

    def __init__(self, n, seed=1, specials=False):
        self.n = n
        self.r = inputs.blackscholes_r(seed, n)
        if specials:  # NaN and +-0 draws (R-RMT4: bitwise compare, no false alarm)
            self.r = inputs.with_specials(self.r, seed, 0.02)
            self.tag = "-specials"

    @functools.cached_property
    def r_d(self):
        return dev(self.r)

    def buffers(self):
        return [self.r_d, out_like(4 * self.n), out_like(4 * self.n)]

    def outputs(self, b):
        return [host(b[1], np.uint32), host(b[2], np.uint32)]

    def check(self, outs, r=None):
        r = self.r if r is None else r
        call_ref, put_ref = oracle.blackscholes(r)
        rr = r.astype(np.float64)
        S = 10 * rr + 100 * (1 - rr)
        nan_in = np.isnan(rr)
        for got_bits, ref in zip(outs, (call_ref, put_ref)):
            got = got_bits.view(np.float32).astype(np.float64)
            assert np.array_equal(np.isnan(got), nan_in), "NaN inputs (only) must give NaN prices"
            # reading R-BS3: relative 1e-4 (BJ tolerance for BlackScholes), floored at 1e-2*S
            tol = 1e-4 * np.maximum(np.abs(ref), 1e-2 * S)
            bad = ~(np.abs(got - ref) <= tol) & ~nan_in
            assert not bad.any(), f"{bad.sum()} mismatches, first at {np.argmax(bad)}"

    def out_elems(self):
        return 1, self.n


class BlackScholesIndep(Case):
    """Independent-parameter mode (dims[0] = 1; reading R-BS4): S != K, so the
    moneyness term ln(S/K) and the x < 0 branch of the CND are exercised."""
    kernel = "blackscholes"

    def __init__(self, n=None, seed=13, edges=False):
        self.prm = inputs.blackscholes_edges() if edges else inputs.blackscholes_indep(seed, n)
        self.n = self.prm.shape[1]
        self.dims = (1,)
        self.tag = "-edges" if edges else "-indep"

    @functools.cached_property
    def p_d(self):
        return dev(self.prm.reshape(-1))

    def buffers(self):
        return [self.p_d, out_like(4 * self.n), out_like(4 * self.n)]

    def outputs(self, b):
        return [host(b[1], np.uint32), host(b[2], np.uint32)]

    def check(self, outs, prm=None):
        prm = self.prm if prm is None else prm
        call, put, cs, ps = oracle.blackscholes_indep(prm)
        scale_floor = 1e-7 * np.maximum(prm[0], prm[1]).astype(np.float64)
        for got_bits, ref, scale in zip(outs, (call, put), (cs, ps)):
            got = got_bits.view(np.float32).astype(np.float64)
            # reading R-BS4: 1e-4 (BJ) relative to the price's two terms |t1| + |t2|
            # (a difference of near-equal terms is ill-conditioned), floored at
            # 1e-7 max(S, K) (~1 fp32 ulp of the price scale)
            bad = ~(np.abs(got - ref) <= 1e-4 * scale + scale_floor)
            assert not bad.any(), f"{bad.sum()} mismatches, first at {np.argmax(bad)}: got {got[bad][:4]} want {ref[bad][:4]}"

    def out_elems(self):
        return 1, self.n


class Reduction(Case):
    kernel = "reduction"

    def __init__(self, n, seed=2, x=None):
        self.n = n
        self.x = inputs.reduction_x(seed, n) if x is None else x

    @functools.cached_property
    def x_d(self):
        return dev(self.x if self.n else np.zeros(4, np.uint32))

    def buffers(self):
        return [self.x_d[: self.n] if self.n else self.x_d[:0], out_like(8)]

    def outputs(self, b):
        return [host(b[1], np.uint64)]

    def check(self, outs, x=None):
        x = self.x if x is None else x
        assert int(outs[0][0]) == oracle.reduction_u32(x)

    def flipped_oracle(self, elem, bit):
        return [np.array([oracle.reduction_u32(_flip(self.x, elem, bit))], np.uint64)]

    def out_elems(self):
        return 1, 1


class Transpose(Case):
    kernel = "transpose"

    def __init__(self, H, W, seed=3, index_coded=False):
        self.H, self.W = H, W
        self.n = H * W
        self.dims = (H, W)
        if index_coded:
            self.A = np.arange(H * W, dtype=np.uint32).reshape(H, W)
        else:
            self.A = inputs.transpose_a(seed, H, W).view(np.uint32)

    @functools.cached_property
    def A_d(self):
        return dev(self.A)

    def buffers(self):
        return [self.A_d, out_like(4 * self.n)]

    def outputs(self, b):
        return [host(b[1], np.uint32).reshape(self.W, self.H)]

    def check(self, outs, A=None):
        A = self.A if A is None else A
        assert np.array_equal(outs[0], oracle.transpose_u32(A))

    def flipped_oracle(self, elem, bit):
        return [oracle.transpose_u32(_flip(self.A, elem, bit))]

    def out_elems(self):
        return 1, self.n


class PrefixSum(Case):
    kernel = "prefixsum"

    def __init__(self, n, seed=4, x=None, exclusive=False, f32=False):
        self.n = n
        self.exclusive, self.f32 = exclusive, f32
        self.dims = (0, 0, (1 if exclusive else 0) | (2 if f32 else 0))
        self.tag = ("-excl" if exclusive else "") + ("-f32" if f32 else "")
        if x is None:
            x = inputs.prefixsum_f32(seed, n) if f32 else inputs.prefixsum_x(seed, n)
        self.x = x

    @functools.cached_property
    def x_d(self):
        return dev(self.x if self.n else np.zeros(4, self.x.dtype))

    def buffers(self):
        y = out_like(4 * max(self.n, 1))[: self.n]
        return [self.x_d[: self.n], y.view(torch.float32) if self.f32 else y]

    def outputs(self, b):
        return [host(b[1], np.uint32)]

    def check(self, outs, x=None):
        x = self.x if x is None else x
        if self.f32:  # fp64 definition, |dy_i| <= 1e-5 sum |x_j| (SURVEY 8(c) PrefixSum fp32 parity rule)
            ref, bound = oracle.prefixsum_f64(x, exclusive=self.exclusive)
            got = outs[0].view(np.float32).astype(np.float64)
            assert np.all(np.abs(got - ref) <= 1e-5 * bound + 1e-30), np.max(np.abs(got - ref) / (bound + 1e-30))
        else:
            assert np.array_equal(outs[0], oracle.prefixsum_u32(x, exclusive=self.exclusive))

    def flipped_oracle(self, elem, bit):
        return [oracle.prefixsum_u32(_flip(self.x, elem, bit))]

    def out_elems(self):
        return 1, self.n


class FWT(Case):
    kernel = "fwt"

    def __init__(self, n, seed=5, ternary=False, specials=False):
        self.n = n
        self.multipass = n > 4096
        self.x = inputs.fwt_ternary(seed, n) if ternary else inputs.fwt_x(seed, n)
        self.specials = specials
        if specials:  # a few +-0 everywhere and one NaN (which spreads to every output)
            self.x = inputs.with_specials(self.x, seed, 0.01, kinds=("+0", "-0"))
            self.x[n // 3] = np.float32(np.nan)
            self.tag = "-specials"

    @functools.cached_property
    def x_d(self):
        return dev(self.x)

    def buffers(self):
        return [self.x_d, out_like(4 * self.n)]

    def outputs(self, b):
        return [host(b[1], np.uint32)]

    def check(self, outs, x=None):
        x = self.x if x is None else x
        if np.isnan(x).any():
            # a NaN reaches every output through the butterflies (payloads differ
            # between CPU and GPU): every output NaN, on both sides
            assert _nan_aware_equal(outs[0], oracle.fwt_f32dag(x).view(np.uint32))
            return
        # R-FWT2: bit-exact vs the fp32 butterfly DAG in the normative stage order
        assert np.array_equal(outs[0], oracle.fwt_f32dag(x).view(np.uint32))
        # and within fp32 rounding of the fp64 definition (BJ 1e-5 relative, scaled by ||x||_1)
        y64 = oracle.fwt_f64(x)
        got = outs[0].view(np.float32).astype(np.float64)
        assert np.max(np.abs(got - y64)) <= 1e-5 * max(1.0, float(np.sum(np.abs(x))) / np.sqrt(len(x)))

    def out_elems(self):
        return 1, self.n

    def flipped_oracle(self, elem, bit):  # R-FWT2: the fp32 DAG is exact
        return [oracle.fwt_f32dag(_flip(self.x, elem, bit)).view(np.uint32)]

    def commit_group(self, e):
        # the final pass's 4-word commit holding word e (k_fwt.cu): the pass-1
        # kernel (N = 4096) commits elements at stride 128, a 7-stage strided pass
        # at stride 2^(s0+5), the generic pass 4 contiguous words
        m = self.n.bit_length() - 1
        if m < 12:
            return super().commit_group(e)
        b = (m - 12) % 7 or 7 if m > 12 else 0
        if m == 12:
            stride = 128
        elif b == 7:
            stride = 1 << (m - 7 + 5)
        else:
            return super().commit_group(e)
        lo = e & ~(3 * stride)
        return lo + stride * np.arange(4)


class BinarySearch(Case):
    kernel = "binarysearch"

    def __init__(self, N, Q, seed=6, odd=False, dups=False, ghost=False):
        self.N, self.Q = N, Q
        self.n = Q
        # ghost: the single-key segment search, one writer per key (dims[2] = 1)
        self.dims = (N, Q, 1) if ghost else (N, Q)
        self.ghost = ghost
        if dups:  # runs of equal keys, 0 and 0xFFFFFFFF in A and in the queries
            self.A, self.q = inputs.binarysearch_dups(seed, N, Q)
            self.tag = "-dups"
        elif odd:
            self.A = (2 * np.arange(N, dtype=np.uint64) + 1).astype(np.uint32)
            self.q = inputs.u32(seed, Q) % np.uint32(2 * N + 8)
        else:
            self.A, self.q = inputs.binarysearch_inputs(seed, max(N, 1), Q)
            self.A = self.A[:N]
        if ghost:
            self.tag += "-ghost"

    @functools.cached_property
    def A_d(self):
        return dev(self.A if self.N else np.zeros(4, np.uint32))[: self.N]

    @functools.cached_property
    def q_d(self):
        return dev(self.q)

    def buffers(self):
        return [self.A_d, self.q_d, out_like(4 * self.Q)]

    def outputs(self, b):
        return [host(b[2], np.uint32)]

    def check(self, outs, A=None, q=None):
        A = self.A if A is None else A
        q = self.q if q is None else q
        assert np.array_equal(outs[0], oracle.binarysearch(A, q))

    def flipped_oracle(self, elem, bit):  # LOAD = the query word
        return [oracle.binarysearch(self.A, _flip(self.q, elem, bit))]

    def commit_group(self, e):
        # a logical thread searches 2 interleaved queries and commits them as one
        # 8-B vector (k_binarysearch.cu); ghost mode commits one word per key
        if self.ghost:
            return np.array([e])
        lo = e - e % 2
        return np.arange(lo, min(lo + 2, self.Q))

    def out_elems(self):
        return 2, self.Q


class Sobel(Case):
    kernel = "sobel"

    def __init__(self, H, W, seed=7, noise=False):
        self.H, self.W = H, W
        self.n = H * W
        self.dims = (H, W)
        if noise:
            self.I = (inputs.u32(seed, H * W * 4) & np.uint32(255)).astype(np.uint8).reshape(H, W, 4)
        else:
            self.I = inputs.sobel_image(seed, H, W)

    @functools.cached_property
    def I_d(self):
        return dev(self.I.view(np.uint32).reshape(-1))

    def buffers(self):
        return [self.I_d, out_like(4 * self.n)]

    def outputs(self, b):
        return [host(b[1], np.uint32)]

    def check(self, outs, I=None):
        I = self.I if I is None else I
        ref = oracle.sobel(I).view(np.uint32).reshape(-1)
        assert np.array_equal(outs[0], ref), f"{np.sum(outs[0] != ref)} pixels differ"

    def flipped_oracle(self, elem, bit):  # LOAD = the 4-channel pixel word
        return [oracle.sobel(_flip(self.I, elem, bit)).view(np.uint32).reshape(-1)]

    def out_elems(self):
        return 1, self.n


class DCT(Case):
    kernel = "dct"

    def __init__(self, H, W, seed=9, specials=False):
        self.H, self.W = H, W
        self.n = H * W
        self.dims = (H, W)
        self.X = inputs.dct_x(seed, H, W)
        if specials:  # NaN and +-0 samples, and one all-(-0) block
            self.X = inputs.with_specials(self.X, seed, 0.002)
            self.X[:8, 8:16] = np.float32(-0.0)
            self.tag = "-specials"

    @functools.cached_property
    def X_d(self):
        return dev(self.X)

    def buffers(self):
        return [self.X_d, out_like(4 * self.n)]

    def outputs(self, b):
        return [host(b[1], np.uint32)]

    def check(self, outs, X=None):
        X = self.X if X is None else X
        H, W = X.shape
        got = outs[0].view(np.float32).reshape(H, W).astype(np.float64)
        ref = oracle.dct8x8(X)
        bound = oracle.dct8x8_absbound(X)
        # NaN inputs: every output of that 8x8 block is NaN on both sides (every
        # DCT-II coefficient C[u][x] is nonzero); the other blocks as usual
        nan = np.isnan(ref)
        assert np.array_equal(np.isnan(got), nan)
        got = np.where(nan, 0.0, got)
        ref = np.where(nan, 0.0, ref)
        bound = np.where(nan, 0.0, bound)
        X = np.where(np.isnan(X), np.float32(0), X)
        # reading R-DCT3: componentwise condition-scaled 1e-5, and per-block normwise 1e-5
        assert np.all(np.abs(got - ref) <= 1e-5 * bound + 1e-30)
        d = (got - ref).reshape(H // 8, 8, W // 8, 8)
        x = X.astype(np.float64).reshape(H // 8, 8, W // 8, 8)
        num = np.sqrt((d ** 2).sum(axis=(1, 3)))
        den = np.sqrt((x ** 2).sum(axis=(1, 3)))
        assert np.all(num <= 1e-5 * np.maximum(den, 1e-30))

    def out_elems(self):
        return 1, self.n


class FloydWarshall(Case):
    kernel = "floydwarshall"

    def __init__(self, n, seed=8, sparse=None):
        self.n = n
        # sparse: edge probability; absent edges = FW_INF (reading R-FW1's secondary graph)
        self.Wm = inputs.floydwarshall_w(seed, n) if sparse is None else inputs.floydwarshall_sparse(seed, n, sparse)
        self.tag = "" if sparse is None else f"-sparse{sparse}"

    @functools.cached_property
    def W_d(self):
        return dev(self.Wm)

    def buffers(self):
        return [self.W_d.clone(), out_like(4 * self.n * self.n)]

    def outputs(self, b):
        return [host(b[0], np.uint32).reshape(self.n, self.n), host(b[1], np.uint32).reshape(self.n, self.n)]

    def check(self, outs, Wm=None):
        Wm = self.Wm if Wm is None else Wm
        D, P = oracle.floydwarshall(Wm)
        assert np.array_equal(outs[0], D)
        assert np.array_equal(outs[1], P)

    def out_elems(self):
        return 0, self.n * self.n

    def fault_target(self, rng):
        # an element whose LAST improving relaxation happens at pass k0: suppressing
        # that store leaves a visibly different final D[e]
        n = self.n
        D = self.Wm.astype(np.int64)
        last = np.full((n, n), -1)
        for k in range(n):
            cand = D[:, k:k + 1] + D[k:k + 1, :]
            better = cand < D
            last[better] = k
            D = np.where(better, cand, D)
        idx = np.flatnonzero(last.reshape(-1) > 0)
        e = int(idx[rng.integers(0, idx.size)])
        k0 = int(last.reshape(-1)[e])
        return k0 * n * n + e, e

    def fault_propagates(self):
        return True

    def commit_group(self, e):
        return np.array([e])  # masked vector commit: only improving words are stored


class MatMul(Case):
    kernel = "matmul"

    def __init__(self, M, N, K, seed=10, integer=False, kc=0):
        self.M, self.N, self.K = M, N, K
        self.n = M * N
        self.dims = (M, N, K, kc)  # kc: TMEM chunk (fold) length in K, 0 = the library default
        self.integer = integer
        if kc:
            self.tag = f"-kc{kc}"
        if integer:
            self.A = inputs.matmul_bf16_int(seed, M, K, stream=20)
            self.Bt = inputs.matmul_bf16_int(seed, N, K, stream=21)
        else:
            self.A = inputs.matmul_bf16_normal(seed, M, K, stream=22)
            self.Bt = inputs.matmul_bf16_normal(seed, N, K, stream=24)

    @functools.cached_property
    def A_d(self):
        return dev(self.A)

    @functools.cached_property
    def B_d(self):
        return dev(self.Bt)

    def buffers(self):
        return [self.A_d, self.B_d, out_like(4 * self.n)]

    def outputs(self, b):
        return [host(b[2], np.uint32).reshape(self.M, self.N)]

    def check(self, outs):
        got = outs[0].view(np.float32).astype(np.float64)
        ref = oracle.matmul_bf16(self.A, self.Bt)
        if self.integer:
            # exactness pin: |partial sums| <= 16 K < 2^24 -> exact in fp32 regardless of order
            assert np.array_equal(got, ref)
            return
        # reading R-MM2: normwise 1e-5, plus the loose elementwise catch-all K 2^-23 (|A||B|)
        assert np.linalg.norm(got - ref) <= 1e-5 * np.linalg.norm(ref)
        Af = np.abs(inputs.bf16_bits_to_f32(self.A).astype(np.float64))
        Bf = np.abs(inputs.bf16_bits_to_f32(self.Bt).astype(np.float64))
        assert np.all(np.abs(got - ref) <= self.K * 2.0 ** -23 * (Af @ Bf.T) + 1e-30)

    def out_elems(self):
        return 2, self.n


class DWT(Case):
    kernel = "dwthaar1d"

    def __init__(self, n, seed=11):
        self.n = n
        self.x = inputs.dwt_x(seed, n)

    @functools.cached_property
    def x_d(self):
        return dev(self.x)

    def buffers(self):
        return [self.x_d, out_like(4 * self.n)]

    def outputs(self, b):
        return [host(b[1], np.uint32)]

    def check(self, outs, x=None):
        x = self.x if x is None else x
        # R-DWT2: bit-exact vs the fp32 DAG in level order
        assert np.array_equal(outs[0], oracle.dwthaar1d_f32dag(x).view(np.uint32))
        # and within 1e-5 of the fp64 definition, scaled by the coefficient's support norm
        y64 = oracle.dwthaar1d_f64(x)
        got = outs[0].view(np.float32).astype(np.float64)
        scale = max(1.0, float(np.sqrt(np.dot(x.astype(np.float64), x))))
        assert np.max(np.abs(got - y64)) <= 1e-5 * scale

    def out_elems(self):
        return 1, self.n

    def flipped_oracle(self, elem, bit):  # R-DWT2: the fp32 DAG is exact
        return [oracle.dwthaar1d_f32dag(_flip(self.x, elem, bit)).view(np.uint32)]


class BitonicSort(Case):
    kernel = "bitonicsort"

    def __init__(self, n, seed=21, bits=32):
        self.n = n
        self.multipass = n > 4096
        self.keys = inputs.bitonic_keys(seed, n, bits=bits)

    @functools.cached_property
    def k_d(self):
        return dev(self.keys)

    def buffers(self):
        return [self.k_d, out_like(4 * self.n)]

    def outputs(self, b):
        return [host(b[1], np.uint32)]

    def check(self, outs, keys=None):
        keys = self.keys if keys is None else keys
        assert np.array_equal(outs[0], oracle.sort_u32(keys))  # R-BIT1: the unique sorted sequence

    def flipped_oracle(self, elem, bit):
        return [oracle.sort_u32(_flip(self.keys, elem, bit))]

    def out_elems(self):
        return 1, self.n


class BinomialOption(Case):
    kernel = "binomialoption"

    def __init__(self, n, seed=12):
        self.n = n
        self.r = inputs.binomial_r(seed, n)

    @functools.cached_property
    def r_d(self):
        return dev(self.r)

    def buffers(self):
        return [self.r_d, out_like(4 * self.n)]

    def outputs(self, b):
        return [host(b[1], np.uint32)]

    def check(self, outs, r=None):
        r = self.r if r is None else r
        ref = oracle.binomialoption(r)
        S = 5.0 * (1 - r.astype(np.float64)) + 30.0 * r.astype(np.float64)
        got = outs[0].view(np.float32).astype(np.float64)
        # reading R-BO2: relative 1e-4 (transcendental + 254-step recurrence, as BlackScholes), floored at 1e-2*S
        bad = ~(np.abs(got - ref) <= 1e-4 * np.maximum(np.abs(ref), 1e-2 * S))
        assert not bad.any(), f"{bad.sum()} mismatches, first at {np.argmax(bad)}"

    def out_elems(self):
        return 1, self.n


def small_cases():
    """Sizes the oracle finishes in seconds that still span several tiles and a ragged tail."""
    return [
        BlackScholes(1), BlackScholes(7), BlackScholes(1024 * 3 + 5), BlackScholes(1 << 16),
        BlackScholes(5003, specials=True),
        BlackScholesIndep(edges=True), BlackScholesIndep(4), BlackScholesIndep(1024 * 3 + 4),
        BlackScholesIndep(1 << 18),
        Reduction(0), Reduction(3), Reduction(1000003), Reduction(1 << 22),
        Transpose(4, 4), Transpose(68, 132), Transpose(256, 512, index_coded=True), Transpose(1000, 764),
        PrefixSum(1), PrefixSum(4095), PrefixSum(4096 * 37 + 11), PrefixSum(1 << 22), PrefixSum((1 << 25) + 12347),
        # the exclusive flag and the fixed-association fp32 scan (SURVEY 8(c) PrefixSum readings (1)-(2))
        PrefixSum(1, exclusive=True), PrefixSum(4096 * 37 + 11, exclusive=True), PrefixSum((1 << 22) + 5, exclusive=True),
        PrefixSum(1, f32=True), PrefixSum(4095, f32=True), PrefixSum(4096 * 37 + 11, f32=True),
        PrefixSum((1 << 22) + 3, f32=True, exclusive=True), PrefixSum(1 << 24, f32=True),
        FWT(1), FWT(2), FWT(64), FWT(4096), FWT(1 << 13), FWT(1 << 19), FWT(1 << 20), FWT(1 << 16, ternary=True),
        FWT(1 << 15, specials=True), FWT(64, specials=True),
        BinarySearch(0, 16), BinarySearch(1, 7), BinarySearch(1000, 1003), BinarySearch(1 << 16, 50000, odd=True),
        BinarySearch(1 << 22, 1 << 18), BinarySearch(15, 100, odd=True), BinarySearch(17, 999),
        BinarySearch((1 << 20) + 13, 70001), BinarySearch(4096 + 9, 5000, odd=True),
        BinarySearch(5, 64, dups=True), BinarySearch(4096 * 3 + 7, 20001, dups=True),
        BinarySearch((1 << 21) + 5, 1 << 16, dups=True),
        # shared-memory table edges (k_binarysearch.cu): n_T = 8192 = P exactly
        # (no padding entry: the final compare), and three sample levels (T = 3)
        BinarySearch(1 << 18, 3001), BinarySearch((8 << 20) + 7, 40000),
        # ghost (single-key segment search): empty A, N < 256 (empty segments), keys past the end, duplicates
        BinarySearch(0, 16, ghost=True), BinarySearch(17, 999, ghost=True), BinarySearch(1000, 1003, ghost=True),
        BinarySearch(1 << 16, 3000, odd=True, ghost=True), BinarySearch(4096 * 3 + 7, 2001, dups=True, ghost=True),
        Sobel(3, 4), Sobel(37, 100), Sobel(100, 1028, noise=True), Sobel(256, 2048),
        DCT(8, 8), DCT(24, 264), DCT(512, 2048 + 8), DCT(64, 512, specials=True),
        FloydWarshall(4), FloydWarshall(52), FloydWarshall(256),
        FloydWarshall(64, sparse=0.03), FloydWarshall(128, sparse=0.1),
        MatMul(128, 256, 64), MatMul(256, 512, 192, integer=True), MatMul(384, 256, 1024),
        MatMul(256, 512, 3072), MatMul(128, 256, 640, kc=64), MatMul(256, 256, 1024, kc=1024),
        MatMul(128, 512, 4096, kc=4096),
        DWT(1), DWT(2), DWT(4), DWT(8), DWT(64), DWT(4096), DWT(8192), DWT(1 << 20), DWT(1 << 23),
        BitonicSort(1), BitonicSort(2), BitonicSort(8), BitonicSort(16), BitonicSort(64, bits=3),
        BitonicSort(4096), BitonicSort(8192, bits=8), BitonicSort(1 << 17), BitonicSort(1 << 20, bits=12),
        BinomialOption(1), BinomialOption(5), BinomialOption(100), BinomialOption(4096 + 3),
    ]
