"""CPU oracle -- TEST INFRASTRUCTURE ONLY.

Plain fp64 / exact-integer definitions of the kernels (oracle.c, which cites
PAPER.md for each).  Only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / `--impl reference` leg may import this package.  The product
path (paper_conf_isca_waddenlgss14_b200) never imports it and shares no code
with it.

Parity status per function: every function here is
pinned by tests/test_oracle_pins.py against closed forms, invariants, brute
force or an independent algorithm; none is "parity unpinned".
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

CFLAGS = ["-O2", "-fopenmp", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared", "-std=gnu11"]


def build(force: bool = False) -> str:
    """Compile oracle.c -> liboracle.so with gcc (plain C, OpenMP)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        P = ctypes.c_void_p
        I = ctypes.c_int64
        D = ctypes.c_double
        L.orc_num_threads.restype = ctypes.c_int
        L.orc_set_threads.argtypes = [ctypes.c_int]
        L.orc_cnd.argtypes = [D]
        L.orc_cnd.restype = D
        L.orc_bs_price.argtypes = [D, D, D, D, D, P, P]
        L.orc_blackscholes.argtypes = [P, I, P, P]
        L.orc_blackscholes_indep.argtypes = [P, I, P, P, P, P]
        L.orc_binarysearch.argtypes = [P, I, P, I, P]
        L.orc_fwt_f64.argtypes = [P, I, P]
        L.orc_fwt_f32dag.argtypes = [P, I, P]
        L.orc_prefixsum_u32.argtypes = [P, I, P]
        L.orc_prefixsum_u32_excl.argtypes = [P, I, P]
        L.orc_prefixsum_f64.argtypes = [P, I, ctypes.c_int, P, P]
        L.orc_reduction_u32.argtypes = [P, I]
        L.orc_reduction_u32.restype = ctypes.c_uint64
        L.orc_transpose_u32.argtypes = [P, I, I, P]
        L.orc_sobel.argtypes = [P, I, I, P]
        L.orc_floydwarshall.argtypes = [P, P, I]
        L.orc_dijkstra_row.argtypes = [P, I, I, P]
        L.orc_dct8x8.argtypes = [P, I, I, P]
        L.orc_dct8x8_absbound.argtypes = [P, I, I, P]
        L.orc_matmul_bf16.argtypes = [P, P, I, I, I, P]
        L.orc_matmul_bf16_sampled.argtypes = [P, P, I, I, P, P, P, P]
        L.orc_sort_u32.argtypes = [P, I, P]
        L.orc_dwthaar1d_f64.argtypes = [P, I, P]
        L.orc_dwthaar1d_f32dag.argtypes = [P, I, P]
        L.orc_crr_price.argtypes = [D, D, D, D, D, I, ctypes.c_int]
        L.orc_crr_price.restype = D
        L.orc_bo_params.argtypes = [D, P, P, P]
        L.orc_binomialoption.argtypes = [P, I, P]
        _lib = L
    return _lib


def _p(a: np.ndarray):
    assert a.flags["C_CONTIGUOUS"]
    return a.ctypes.data_as(ctypes.c_void_p)


def num_threads() -> int:
    return lib().orc_num_threads()


def set_threads(n: int) -> None:
    lib().orc_set_threads(int(n))


def cnd(x: float) -> float:
    return lib().orc_cnd(float(x))


def bs_price(S, K, T, R, V):
    c = ctypes.c_double()
    p = ctypes.c_double()
    lib().orc_bs_price(S, K, T, R, V, ctypes.byref(c), ctypes.byref(p))
    return c.value, p.value


def blackscholes(r: np.ndarray):
    r = np.ascontiguousarray(r, dtype=np.float32)
    call = np.empty(r.size, np.float64)
    put = np.empty(r.size, np.float64)
    lib().orc_blackscholes(_p(r), r.size, _p(call), _p(put))
    return call, put


def blackscholes_indep(prm: np.ndarray):
    """prm: float32 (5, n) planes S, K, T, R, sigma -> (call, put, call_scale, put_scale)."""
    prm = np.ascontiguousarray(prm, dtype=np.float32)
    assert prm.ndim == 2 and prm.shape[0] == 5
    n = prm.shape[1]
    out = [np.empty(n, np.float64) for _ in range(4)]
    lib().orc_blackscholes_indep(_p(prm), n, *[_p(o) for o in out])
    return tuple(out)


def binarysearch(A: np.ndarray, q: np.ndarray) -> np.ndarray:
    A = np.ascontiguousarray(A, dtype=np.uint32)
    q = np.ascontiguousarray(q, dtype=np.uint32)
    idx = np.empty(q.size, np.uint32)
    lib().orc_binarysearch(_p(A), A.size, _p(q), q.size, _p(idx))
    return idx


def fwt_f64(x: np.ndarray) -> np.ndarray:
    x = np.ascontiguousarray(x, dtype=np.float32)
    y = np.empty(x.size, np.float64)
    lib().orc_fwt_f64(_p(x), x.size, _p(y))
    return y


def fwt_f32dag(x: np.ndarray) -> np.ndarray:
    x = np.ascontiguousarray(x, dtype=np.float32)
    y = np.empty(x.size, np.float32)
    lib().orc_fwt_f32dag(_p(x), x.size, _p(y))
    return y


def prefixsum_u32(x: np.ndarray, exclusive: bool = False) -> np.ndarray:
    x = np.ascontiguousarray(x, dtype=np.uint32)
    y = np.empty(x.size, np.uint32)
    (lib().orc_prefixsum_u32_excl if exclusive else lib().orc_prefixsum_u32)(_p(x), x.size, _p(y))
    return y


def prefixsum_f64(x: np.ndarray, exclusive: bool = False):
    """fp64 scan of fp32 inputs and its conditioning bound sum |x_j| (oracle.c)."""
    x = np.ascontiguousarray(x, dtype=np.float32)
    y = np.empty(x.size, np.float64)
    b = np.empty(x.size, np.float64)
    lib().orc_prefixsum_f64(_p(x), x.size, 1 if exclusive else 0, _p(y), _p(b))
    return y, b


def reduction_u32(x: np.ndarray) -> int:
    x = np.ascontiguousarray(x, dtype=np.uint32)
    return int(lib().orc_reduction_u32(_p(x), x.size))


def transpose_u32(A: np.ndarray) -> np.ndarray:
    A = np.ascontiguousarray(A)
    H, W = A.shape
    a32 = A.view(np.uint32)
    B = np.empty((W, H), np.uint32)
    lib().orc_transpose_u32(_p(a32), H, W, _p(B))
    return B.view(A.dtype)


def sobel(I: np.ndarray) -> np.ndarray:
    I = np.ascontiguousarray(I, dtype=np.uint8)
    H, W, C = I.shape
    assert C == 4
    O = np.empty_like(I)
    lib().orc_sobel(_p(I), H, W, _p(O))
    return O


def floydwarshall(Wm: np.ndarray):
    n = Wm.shape[0]
    D = np.ascontiguousarray(Wm, dtype=np.uint32).copy()
    P = np.repeat(np.arange(n, dtype=np.uint32)[:, None], n, axis=1).copy()  # R-FW2: P[i][j] = i
    lib().orc_floydwarshall(_p(D), _p(P), n)
    return D, P


def dijkstra_row(Wm: np.ndarray, src: int) -> np.ndarray:
    Wm = np.ascontiguousarray(Wm, dtype=np.uint32)
    n = Wm.shape[0]
    d = np.empty(n, np.uint32)
    lib().orc_dijkstra_row(_p(Wm), n, int(src), _p(d))
    return d


def dct8x8(X: np.ndarray) -> np.ndarray:
    X = np.ascontiguousarray(X, dtype=np.float32)
    H, W = X.shape
    Y = np.empty((H, W), np.float64)
    lib().orc_dct8x8(_p(X), H, W, _p(Y))
    return Y


def dct8x8_absbound(X: np.ndarray) -> np.ndarray:
    X = np.ascontiguousarray(X, dtype=np.float32)
    H, W = X.shape
    Y = np.empty((H, W), np.float64)
    lib().orc_dct8x8_absbound(_p(X), H, W, _p(Y))
    return Y


def matmul_bf16(A: np.ndarray, Bt: np.ndarray) -> np.ndarray:
    A = np.ascontiguousarray(A, dtype=np.uint16)
    Bt = np.ascontiguousarray(Bt, dtype=np.uint16)
    M, K = A.shape
    N, K2 = Bt.shape
    assert K == K2
    C = np.empty((M, N), np.float64)
    lib().orc_matmul_bf16(_p(A), _p(Bt), M, N, K, _p(C))
    return C


def matmul_bf16_sampled(A: np.ndarray, Bt: np.ndarray, rows: np.ndarray, cols: np.ndarray):
    A = np.ascontiguousarray(A, dtype=np.uint16)
    Bt = np.ascontiguousarray(Bt, dtype=np.uint16)
    rows = np.ascontiguousarray(rows, dtype=np.int64)
    cols = np.ascontiguousarray(cols, dtype=np.int64)
    out = np.empty(rows.size, np.float64)
    absout = np.empty(rows.size, np.float64)
    lib().orc_matmul_bf16_sampled(_p(A), _p(Bt), A.shape[1], rows.size, _p(rows), _p(cols),
                                  _p(out), _p(absout))
    return out, absout


def sort_u32(keys: np.ndarray) -> np.ndarray:
    keys = np.ascontiguousarray(keys, dtype=np.uint32)
    out = np.empty_like(keys)
    lib().orc_sort_u32(_p(keys), keys.size, _p(out))
    return out


def dwthaar1d_f64(x: np.ndarray) -> np.ndarray:
    x = np.ascontiguousarray(x, dtype=np.float32)
    y = np.empty(x.size, np.float64)
    lib().orc_dwthaar1d_f64(_p(x), x.size, _p(y))
    return y


def dwthaar1d_f32dag(x: np.ndarray) -> np.ndarray:
    x = np.ascontiguousarray(x, dtype=np.float32)
    y = np.empty(x.size, np.float32)
    lib().orc_dwthaar1d_f32dag(_p(x), x.size, _p(y))
    return y


BO_STEPS, BO_R, BO_V = 254, 0.02, 0.30


def crr_price(S, K, T, R, V, N, call=True) -> float:
    return lib().orc_crr_price(float(S), float(K), float(T), float(R), float(V), int(N), 1 if call else 0)


def bo_params(r: float):
    S, K, T = ctypes.c_double(), ctypes.c_double(), ctypes.c_double()
    lib().orc_bo_params(float(r), ctypes.byref(S), ctypes.byref(K), ctypes.byref(T))
    return S.value, K.value, T.value


def binomialoption(r: np.ndarray) -> np.ndarray:
    r = np.ascontiguousarray(r, dtype=np.float32)
    call = np.empty(r.size, np.float64)
    lib().orc_binomialoption(_p(r), r.size, _p(call))
    return call
