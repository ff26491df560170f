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

    def commit_group(self, e):
        """Word indices of the first output buffer stored by the same commit as
        word e (one commit per store instruction; vector stores are 4 words)."""
        b, ne = self.out_elems()
        lo = e - e % 4
        return np.arange(lo, min(lo + 4, ne))


class BlackScholes(Case):
    kernel = "blackscholes"

    def __init__(self, n, seed=1):
        self.n = n
        self.r = inputs.blackscholes_r(seed, n)

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
        for got_bits, ref in zip(outs, (call_ref, put_ref)):
            got = got_bits.view(np.float32).astype(np.float64)
            # reading R-BS3: relative 1e-4 (BJ tolerance for BlackScholes), floored at 1e-2*S
            tol = 1e-4 * np.maximum(np.abs(ref), 1e-2 * S)
            bad = ~(np.abs(got - ref) <= tol)
            assert not bad.any(), f"{bad.sum()} mismatches, first at {np.argmax(bad)}"

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

    def out_elems(self):
        return 1, self.n


def small_cases():
    """Sizes the oracle finishes in seconds that still span several tiles and a ragged tail."""
    return [
        BlackScholes(1), BlackScholes(7), BlackScholes(1024 * 3 + 5), BlackScholes(1 << 16),
        Reduction(0), Reduction(3), Reduction(1000003), Reduction(1 << 22),
        Transpose(4, 4), Transpose(68, 132), Transpose(256, 512, index_coded=True), Transpose(1000, 764),
    ]
