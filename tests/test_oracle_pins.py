"""Pins for the CPU oracle (-m "not gpu").

Each test checks the oracle against something other than itself: a closed
form, an invariant, brute force on a tiny input, an independent algorithm or
a library routine the definition reduces to.  A
plausible mistake anywhere in oracle.c (dropped term, wrong sign or index,
transposed operand) must fail one of these.
"""
import itertools
import math

import numpy as np
import pytest
import scipy.fft
import scipy.ndimage

import oracle
from paper_conf_isca_waddenlgss14_b200 import inputs

# ---------------------------------------------------------------- BlackScholes


def test_cnd_matches_erfc_within_as_bound():
    # A&S 26.2.17 has |error| < 7.5e-8 against the exact normal CDF.
    for x in np.linspace(-8, 8, 4001):
        exact = 0.5 * math.erfc(-x / math.sqrt(2.0))
        assert abs(oracle.cnd(x) - exact) < 7.5e-8, x


def test_cnd_symmetry():
    # N(-x) = 1 - N(x) holds by construction for x != 0; at 0 the polynomial
    # itself is off by its A&S error (5e-10).
    for x in np.linspace(-5, 5, 100):
        assert abs(oracle.cnd(x) + oracle.cnd(-x) - 1.0) < 1e-15
    assert abs(oracle.cnd(0.0) - 0.5) < 7.5e-8


def test_bs_textbook_point():
    # Hull, Options Futures & Other Derivatives: S=K=100, T=1, r=5%, sigma=20%
    c, p = oracle.bs_price(100.0, 100.0, 1.0, 0.05, 0.2)
    assert abs(c - 10.45058) < 1e-4
    assert abs(p - 5.57353) < 1e-4


def _bs_exact(S, K, T, R, V):
    N = lambda x: 0.5 * math.erfc(-x / math.sqrt(2.0))
    d1 = (math.log(S / K) + (R + V * V / 2) * T) / (V * math.sqrt(T))
    d2 = d1 - V * math.sqrt(T)
    return S * N(d1) - K * math.exp(-R * T) * N(d2), K * math.exp(-R * T) * N(-d2) - S * N(-d1)


def test_bs_workload_mapping_and_exact_price():
    # R-BS1 mapping at r=0 and r=1 and a sample of draws, against the exact-erfc
    # price; the A&S error bound gives |dC| <= 2*7.5e-8*(S+K).
    r = inputs.blackscholes_r(7, 2000)
    r = np.concatenate([r, np.array([0.0, 1.0 - 2**-24], np.float32)])
    call, put = oracle.blackscholes(r)
    for i, ri in enumerate(r.astype(np.float64)):
        S = 10 * ri + 100 * (1 - ri)
        T = 1 * ri + 10 * (1 - ri)
        R = 0.01 * ri + 0.05 * (1 - ri)
        V = 0.01 * ri + 0.10 * (1 - ri)
        ce, pe = _bs_exact(S, S, T, R, V)
        assert abs(call[i] - ce) <= 3e-7 * S
        assert abs(put[i] - pe) <= 3e-7 * S


def test_bs_indep_printed_values():
    # printed textbook values through the independent-parameter path (R-BS4):
    # Hull's ATM point and Hull Example 15.6 (S=42, K=40, T=0.5, r=10%, sigma=20%:
    # c = 4.76, p = 0.81 to the printed 2 decimals)
    prm = inputs.blackscholes_edges()
    call, put, _, _ = oracle.blackscholes_indep(prm)
    assert abs(call[0] - 10.45058) < 1e-4 and abs(put[0] - 5.57353) < 1e-4
    assert round(call[1], 2) == 4.76 and round(put[1], 2) == 0.81


def test_bs_indep_exact_parity_bounds_scale():
    # independent draws: S != K, d1/d2 of both signs, deep ITM/OTM
    prm = np.concatenate([inputs.blackscholes_indep(21, 5000), inputs.blackscholes_edges()], axis=1)
    call, put, cs, ps = oracle.blackscholes_indep(prm)
    S, K, T, R, V = (prm[k].astype(np.float64) for k in range(5))
    disc = K * np.exp(-R * T)
    d1 = (np.log(S / K) + (R + V * V / 2) * T) / (V * np.sqrt(T))
    assert (d1 < -1).any() and (d1 > 1).any() and (d1 - V * np.sqrt(T) < 0).any()  # both CND branches
    # put-call parity (exact for any N with N(-x) = 1 - N(x)), and the no-arbitrage bounds
    assert np.max(np.abs(call - put - (S - disc)) / np.maximum(S, K)) < 1e-12
    assert np.all(call >= np.maximum(0, S - disc) - 1e-9) and np.all(call <= S + 1e-9)
    assert np.all(put >= np.maximum(0, disc - S) - 1e-9) and np.all(put <= disc + 1e-9)
    # against the exact-erfc price (a different CND): the A&S bound 7.5e-8 per N
    for i in range(0, prm.shape[1], 7):
        ce, pe = _bs_exact(S[i], K[i], T[i], R[i], V[i])
        assert abs(call[i] - ce) <= 7.5e-8 * (S[i] + disc[i]) + 1e-12
        assert abs(put[i] - pe) <= 7.5e-8 * (S[i] + disc[i]) + 1e-12
    # the conditioning scales bound the prices and the terms
    assert np.all(cs >= np.abs(call) - 1e-12) and np.all(ps >= np.abs(put) - 1e-12)
    assert np.all(cs <= S + disc + 1e-9) and np.all(ps <= S + disc + 1e-9)
    # deep OTM call underflows, deep ITM call = S - K e^{-RT} to within the tail
    i_otm, i_itm = 3, 7  # BS_EDGE_ROWS: (5, 100, .25, .01, .1) and (5, 1, .25, .05, .1)
    assert call[prm.shape[1] - inputs.blackscholes_edges().shape[1] + i_otm] < 1e-30
    j = prm.shape[1] - inputs.blackscholes_edges().shape[1] + i_itm
    assert abs(call[j] - (S[j] - disc[j])) < 1e-9


def test_bs_put_call_parity_and_bounds():
    r = inputs.blackscholes_r(3, 1 << 16)
    call, put = oracle.blackscholes(r)
    rr = r.astype(np.float64)
    S = 10 * rr + 100 * (1 - rr)
    T = 1 * rr + 10 * (1 - rr)
    R = 0.01 * rr + 0.05 * (1 - rr)
    disc = S * np.exp(-R * T)
    assert np.max(np.abs(call - put - (S - disc))) < 1e-10 * 100
    assert np.all(call >= np.maximum(0, S - disc) - 1e-9) and np.all(call <= S)
    assert np.all(put >= np.maximum(0, disc - S) - 1e-9) and np.all(put <= disc)


# ---------------------------------------------------------------- BinarySearch


def test_binarysearch_closed_form_odd_numbers():
    N = 1 << 16
    A = (2 * np.arange(N, dtype=np.uint64) + 1).astype(np.uint32)
    q = np.concatenate([np.arange(0, 2 * N + 8, dtype=np.uint32),
                        inputs.u32(1, 4096)])
    idx = oracle.binarysearch(A, q)
    expect = np.minimum(N, q.astype(np.uint64) // 2)
    assert np.array_equal(idx.astype(np.uint64), expect)


def test_binarysearch_brute_force_tiny():
    for N in [1, 2, 3, 7, 64]:
        A, q = inputs.binarysearch_inputs(11 + N, N, 300)
        q = np.concatenate([q, A, A + 1, np.array([0, 2**32 - 1], np.uint32)])
        idx = oracle.binarysearch(A, q)
        brute = np.array([(A < k).sum() for k in q], np.uint32)
        assert np.array_equal(idx, brute)


def test_binarysearch_vs_searchsorted():
    A, q = inputs.binarysearch_inputs(5, 1 << 18, 1 << 16)
    assert np.all(A[1:] > A[:-1])
    assert np.array_equal(oracle.binarysearch(A, q), np.searchsorted(A, q, side="left").astype(np.uint32))


def test_binarysearch_duplicates_and_extremes():
    # runs of equal keys, 0 and 0xFFFFFFFF in A and in q: lower_bound is the
    # first index of the run (brute-force count and numpy's side="left")
    for N, Q in [(1, 50), (5, 64), (300, 2000), (1 << 16, 1 << 14)]:
        A, q = inputs.binarysearch_dups(N, N, Q)
        assert np.all(A[1:] >= A[:-1]) and (N < 8 or (A[1:] == A[:-1]).any())
        idx = oracle.binarysearch(A, q)
        assert np.array_equal(idx, np.searchsorted(A, q, side="left").astype(np.uint32))
        if N <= 300:
            assert np.array_equal(idx, np.array([(A < k).sum() for k in q], np.uint32))
        # found <=> A[idx] == key, and then idx is the first of its run
        f = idx < N
        hit = f.copy()
        hit[f] = A[idx[f]] == q[f]
        assert np.all((idx[hit] == 0) | (A[np.maximum(idx[hit].astype(np.int64) - 1, 0)] < q[hit]))
    A = np.full(10, 0xFFFFFFFF, np.uint32)
    assert list(oracle.binarysearch(A, np.array([0, 0xFFFFFFFE, 0xFFFFFFFF], np.uint32))) == [0, 0, 0]
    A = np.zeros(10, np.uint32)
    assert list(oracle.binarysearch(A, np.array([0, 1, 0xFFFFFFFF], np.uint32))) == [0, 10, 10]


# ---------------------------------------------------------------- FastWalshTransform


def _hadamard(N):
    i = np.arange(N)
    pc = np.vectorize(lambda v: bin(v).count("1"))(i[:, None] & i[None, :])
    return np.where(pc % 2 == 0, 1, -1).astype(np.int64)


def test_fwt_brute_force_matrix():
    for N in [1, 2, 4, 64, 1024]:
        x = inputs.fwt_x(2, N)
        y = oracle.fwt_f64(x)
        ref = _hadamard(N).astype(np.float64) @ x.astype(np.float64)
        assert np.allclose(y, ref, rtol=0, atol=1e-9 * max(1, N))


def test_fwt_exact_integer_pin_f32dag():
    # x in {-1,0,1}: every partial sum is an integer of magnitude <= N <= 2^24,
    # so the fp32 DAG is exact and equals the int64 transform bit for bit.
    N = 4096
    x = inputs.fwt_ternary(9, N)
    y32 = oracle.fwt_f32dag(x)
    ref = _hadamard(N) @ x.astype(np.int64)
    assert np.array_equal(y32.astype(np.int64), ref)
    # involution: H(H x) = N x (exact, integers)
    yy = oracle.fwt_f32dag(y32)
    assert np.array_equal(yy.astype(np.int64), N * x.astype(np.int64))


def test_fwt_delta_and_parseval():
    N = 1 << 12
    j = 1234
    x = np.zeros(N, np.float32)
    x[j] = 1
    y = oracle.fwt_f64(x)
    expect = np.array([(-1) ** bin(i & j).count("1") for i in range(N)], np.float64)
    assert np.array_equal(y, expect)
    x = inputs.fwt_x(4, 1 << 16)
    y = oracle.fwt_f64(x)
    assert abs(np.sum(y * y) / (len(x) * np.sum(x.astype(np.float64) ** 2)) - 1) < 1e-12
    # the fp32 DAG stays within fp32 rounding of the fp64 transform
    y32 = oracle.fwt_f32dag(x).astype(np.float64)
    assert np.max(np.abs(y32 - y)) <= 16 * 2.0**-24 * np.sum(np.abs(x))


# ---------------------------------------------------------------- PrefixSum / Reduction


def test_prefixsum_closed_forms():
    n = 1 << 17
    ones = np.ones(n, np.uint32)
    assert np.array_equal(oracle.prefixsum_u32(ones), np.arange(1, n + 1, dtype=np.uint32))
    i = np.arange(n, dtype=np.uint64)
    y = oracle.prefixsum_u32(i.astype(np.uint32))
    assert np.array_equal(y, ((i * (i + 1) // 2) % 2**32).astype(np.uint32))


def test_prefixsum_differencing_and_library():
    x = inputs.prefixsum_x(3, 100003)
    y = oracle.prefixsum_u32(x)
    d = np.diff(y.astype(np.int64)) % 2**32
    assert np.array_equal(d, x[1:].astype(np.int64)) and y[0] == x[0]
    assert np.array_equal(y, np.cumsum(x, dtype=np.uint32))


def test_prefixsum_exclusive_closed_forms():
    """Exclusive scan (SURVEY 8(c) PrefixSum reading (1)): x = 1 -> y_i = i;
    x_i = i -> i(i-1)/2 mod 2^32; y_0 = 0; differences recover the input."""
    n = 1 << 17
    assert np.array_equal(oracle.prefixsum_u32(np.ones(n, np.uint32), exclusive=True), np.arange(n, dtype=np.uint32))
    i = np.arange(n, dtype=np.uint64)
    y = oracle.prefixsum_u32(i.astype(np.uint32), exclusive=True)
    assert np.array_equal(y, ((i * (i - 1) // 2) % 2**32).astype(np.uint32))
    x = inputs.prefixsum_x(4, 50001)
    y = oracle.prefixsum_u32(x, exclusive=True)
    assert y[0] == 0 and np.array_equal(np.diff(y.astype(np.int64)) % 2**32, x[:-1].astype(np.int64))
    assert oracle.prefixsum_u32(np.zeros(0, np.uint32), exclusive=True).size == 0


def test_prefixsum_f64_closed_forms_and_library():
    """fp64 oracle of the fp32 scan: integer-valued inputs are exact (x = 1 ->
    i + 1; alternating +-1 -> 1, 0, 1, 0, ...), random inputs equal numpy's fp64
    cumulative sum to the last bit of a few ulps, the bound is the cumulative sum
    of |x|, exclusive is the shift with y_0 = b_0 = 0."""
    n = 100003
    y, b = oracle.prefixsum_f64(np.ones(n, np.float32))
    assert np.array_equal(y, np.arange(1, n + 1, dtype=np.float64)) and np.array_equal(b, y)
    alt = np.where(np.arange(n) % 2 == 0, 1.0, -1.0).astype(np.float32)
    y, b = oracle.prefixsum_f64(alt)
    assert np.array_equal(y, (np.arange(n) % 2 == 0).astype(np.float64))
    assert np.array_equal(b, np.arange(1, n + 1, dtype=np.float64))
    rng = np.random.default_rng(9)
    x = rng.uniform(-1, 1, n).astype(np.float32)
    y, b = oracle.prefixsum_f64(x)
    ref = np.cumsum(x.astype(np.float64))
    assert np.max(np.abs(y - ref)) <= 1e-9
    assert np.allclose(b, np.cumsum(np.abs(x.astype(np.float64))), rtol=1e-12)
    ye, be = oracle.prefixsum_f64(x, exclusive=True)
    assert ye[0] == 0.0 and be[0] == 0.0 and np.array_equal(ye[1:], y[:-1]) and np.array_equal(be[1:], b[:-1])


def test_reduction_closed_forms():
    n = (1 << 20) + 37
    assert oracle.reduction_u32(np.full(n, 7, np.uint32)) == 7 * n
    i = np.arange(n, dtype=np.uint64)
    x = (i % 65536).astype(np.uint32)
    full, rem = divmod(n, 65536)
    expect = full * (65535 * 65536 // 2) + rem * (rem - 1) // 2
    assert oracle.reduction_u32(x) == expect
    x = inputs.reduction_x(2, n)
    assert oracle.reduction_u32(x) == int(np.sum(x, dtype=np.uint64))
    assert oracle.reduction_u32(x) % 2**32 == int(oracle.prefixsum_u32(x)[-1])
    assert oracle.reduction_u32(np.zeros(0, np.uint32)) == 0


# ---------------------------------------------------------------- Transpose


def test_transpose_index_coded_and_involution():
    H, W = 96, 200
    A = np.arange(H * W, dtype=np.uint32).reshape(H, W)
    B = oracle.transpose_u32(A)
    jj, ii = np.meshgrid(np.arange(H), np.arange(W))
    assert np.array_equal(B, (jj * W + ii).astype(np.uint32))
    assert np.array_equal(oracle.transpose_u32(B), A)
    X = inputs.transpose_a(1, 33, 65)
    assert np.array_equal(oracle.transpose_u32(X), X.T)


# ---------------------------------------------------------------- Sobel


def _sobel_scipy(I):
    # independent: scipy correlate with the two 3x3 masks (rows = dy, cols = dx)
    kx = np.array([[1, 2, 1], [0, 0, 0], [-1, -2, -1]])
    ky = np.array([[1, 0, -1], [2, 0, -2], [1, 0, -1]])
    out = np.zeros_like(I)
    for c in range(4):
        ch = I[:, :, c].astype(np.int64)
        gx = scipy.ndimage.correlate(ch, kx, mode="constant")
        gy = scipy.ndimage.correlate(ch, ky, mode="constant")
        m = np.floor(np.sqrt((gx * gx + gy * gy).astype(np.float64))).astype(np.int64) // 2
        o = np.minimum(255, m)
        o[0, :] = o[-1, :] = 0
        o[:, 0] = o[:, -1] = 0
        out[:, :, c] = o
    return out


def test_sobel_vs_scipy_correlate():
    I = inputs.sobel_image(3, 70, 131)
    assert np.array_equal(oracle.sobel(I), _sobel_scipy(I))
    rnd = (inputs.u32(8, 40 * 50 * 4) & 255).astype(np.uint8).reshape(40, 50, 4)
    assert np.array_equal(oracle.sobel(rnd), _sobel_scipy(rnd))


def test_sobel_closed_forms():
    H, W = 16, 24
    assert not oracle.sobel(np.full((H, W, 4), 77, np.uint8)).any()
    for a in [1, 3, 9]:
        x = np.arange(W)
        I = np.broadcast_to((a * x)[None, :, None], (H, W, 4)).astype(np.uint8)
        O = oracle.sobel(I)
        assert np.all(O[1:-1, 1:-1] == min(255, 4 * a))
        assert not O[0].any() and not O[:, 0].any()
    I = np.zeros((H, W, 4), np.uint8)
    I[5, 7, 2] = 200
    O = oracle.sobel(I)
    # diagonal neighbour sees |Gx| = |Gy| = 200 -> floor(sqrt(2)*200)//2 = 141
    assert O[6, 8, 2] == math.isqrt(2 * 200 * 200) // 2
    # side neighbour sees one gradient of 2*200 -> 200
    assert O[5, 8, 2] == 200
    assert O[5, 7, 2] == 0 and not O[:, :, [0, 1, 3]].any()


# ---------------------------------------------------------------- FloydWarshall


def test_floydwarshall_vs_dijkstra_and_invariants():
    n = 96
    Wm = inputs.floydwarshall_w(4, n)
    D, P = oracle.floydwarshall(Wm)
    for s in [0, 5, 50, 95]:
        assert np.array_equal(D[s], oracle.dijkstra_row(Wm, s))
    assert not np.diag(D).any()
    assert np.all(D <= Wm)
    # path invariant: P[i][j] = i  =>  D = W ; else D[i][j] = D[i][p] + D[p][j]
    for i in range(n):
        for j in range(n):
            p = P[i, j]
            if p == i:
                assert D[i, j] == Wm[i, j]
            else:
                assert D[i, j] == D[i, p] + D[p, j]
    # triangle inequality
    for i, j, k in itertools.product(range(0, n, 7), repeat=3):
        assert D[i, j] <= D[i, k] + D[k, j]


def test_floydwarshall_brute_force_paths_tiny():
    n = 6
    Wm = inputs.floydwarshall_w(12, n)
    D, _ = oracle.floydwarshall(Wm)
    for i in range(n):
        for j in range(n):
            best = int(Wm[i, j]) if i != j else 0
            others = [v for v in range(n) if v not in (i, j)]
            for L in range(1, len(others) + 1):
                for mid in itertools.permutations(others, L):
                    path = (i,) + mid + (j,)
                    best = min(best, sum(int(Wm[a, b]) for a, b in zip(path, path[1:])))
            assert D[i, j] == best


def test_floydwarshall_sparse_inf_edges():
    # absent edges = FW_INF (R-FW1 secondary graph): D rows against Dijkstra,
    # unreachable pairs keep exactly FW_INF with P = i, brute force on n = 6
    n = 80
    Wm = inputs.floydwarshall_sparse(3, n, 0.03)
    D, P = oracle.floydwarshall(Wm)
    for s in [0, 1, 40, 79]:
        assert np.array_equal(D[s], oracle.dijkstra_row(Wm, s))
    unreach = D >= inputs.FW_INF
    assert unreach.any() and (~unreach).sum() > n
    assert np.all(D[unreach] == inputs.FW_INF)
    rows = np.repeat(np.arange(n, dtype=np.uint32)[:, None], n, axis=1)
    assert np.array_equal(P[unreach], rows[unreach])
    n = 6
    Wm = inputs.floydwarshall_sparse(5, n, 0.4)
    D, _ = oracle.floydwarshall(Wm)
    for i in range(n):
        for j in range(n):
            best = int(Wm[i, j]) if i != j else 0
            others = [v for v in range(n) if v not in (i, j)]
            for L in range(1, len(others) + 1):
                for mid in itertools.permutations(others, L):
                    path = (i,) + mid + (j,)
                    best = min(best, sum(int(Wm[a, b]) for a, b in zip(path, path[1:])))
            assert D[i, j] == best


def test_floydwarshall_pred_is_last_strict_improvement():
    # strict '<': with all-equal weights nothing ever improves -> P stays i
    n = 10
    Wm = np.full((n, n), 5, np.uint32)
    np.fill_diagonal(Wm, 0)
    D, P = oracle.floydwarshall(Wm)
    assert np.array_equal(D, Wm)
    assert np.array_equal(P, np.repeat(np.arange(n, dtype=np.uint32)[:, None], n, axis=1))


# ---------------------------------------------------------------- DCT


def test_dct_vs_scipy_and_closed_forms():
    X = inputs.dct_x(5, 32, 48)
    Y = oracle.dct8x8(X)
    for by in range(4):
        for bx in range(6):
            blk = X[by * 8:(by + 1) * 8, bx * 8:(bx + 1) * 8].astype(np.float64)
            ref = scipy.fft.dctn(blk, type=2, norm="ortho")
            got = Y[by * 8:(by + 1) * 8, bx * 8:(bx + 1) * 8]
            assert np.allclose(got, ref, rtol=0, atol=1e-10)
            assert abs(np.linalg.norm(got) - np.linalg.norm(blk)) < 1e-9  # Parseval
    c = 3.5
    Yc = oracle.dct8x8(np.full((8, 8), c, np.float32))
    assert abs(Yc[0, 0] - 8 * c) < 1e-12 and np.max(np.abs(Yc.ravel()[1:])) < 1e-12
    # basis: X = C[u]^T C[v] -> Y = e_uv
    u, v = 3, 5
    Cm = np.array([[(math.sqrt(1 / 8) if a == 0 else 0.5) * math.cos((2 * x + 1) * a * math.pi / 16)
                    for x in range(8)] for a in range(8)])
    Xb = np.outer(Cm[u], Cm[v]).astype(np.float32)
    Yb = oracle.dct8x8(Xb)
    E = np.zeros((8, 8))
    E[u, v] = 1
    assert np.allclose(Yb, E, atol=1e-6)
    B = oracle.dct8x8_absbound(X)
    assert np.all(B >= np.abs(Y) - 1e-9)


def test_dct_absbound_tight_and_additive():
    """The conditioning bound B[u][v] = sum_xy |C[u][x]| |X[x][y]| |C[v][y]| is
    pinned by what it must satisfy, not by its formula: on a delta block every
    Y[u][v] is a single product, so B == |Y| exactly; B is additive over
    blocks of disjoint support and absolutely homogeneous; a sign-matched block
    X = outer(sign C[u], sign C[v]) attains B[u][v] = |Y[u][v]|."""
    Cm = np.array([[(math.sqrt(1 / 8) if a == 0 else 0.5) * math.cos((2 * x + 1) * a * math.pi / 16)
                    for x in range(8)] for a in range(8)])
    Bsum = np.zeros((8, 8))
    rng = np.random.default_rng(5)
    Xr = rng.uniform(-3, 3, (8, 8)).astype(np.float32)
    for x in range(8):
        for y in range(8):
            D = np.zeros((8, 8), np.float32)
            D[x, y] = 1.0
            Bd = oracle.dct8x8_absbound(D)
            assert np.allclose(Bd, np.abs(oracle.dct8x8(D)), rtol=1e-12, atol=1e-15)
            Bsum += abs(float(Xr[x, y])) * Bd
    assert np.allclose(oracle.dct8x8_absbound(Xr), Bsum, rtol=1e-12, atol=1e-12)
    assert np.allclose(oracle.dct8x8_absbound(-2 * Xr), 2 * oracle.dct8x8_absbound(Xr), rtol=1e-12)
    for u, v in ((0, 0), (3, 5), (7, 1)):
        Xs = np.outer(np.sign(Cm[u]), np.sign(Cm[v])).astype(np.float32)
        assert abs(oracle.dct8x8_absbound(Xs)[u, v] - abs(oracle.dct8x8(Xs)[u, v])) < 1e-9


# ---------------------------------------------------------------- MatrixMultiplication


def test_matmul_integer_exact_vs_numpy():
    M, N, K = 64, 48, 96
    A = inputs.matmul_bf16_int(1, M, K, stream=20)
    Bt = inputs.matmul_bf16_int(1, N, K, stream=21)
    Af = inputs.bf16_bits_to_f32(A).astype(np.int64)
    Bf = inputs.bf16_bits_to_f32(Bt).astype(np.int64)
    C = oracle.matmul_bf16(A, Bt)
    assert np.array_equal(C.astype(np.int64), Af @ Bf.T)


def test_matmul_normal_vs_numpy_and_freivalds_and_samples():
    M, N, K = 40, 56, 72
    A = inputs.matmul_bf16_normal(2, M, K, stream=22)
    Bt = inputs.matmul_bf16_normal(2, N, K, stream=24)
    Af = inputs.bf16_bits_to_f32(A).astype(np.float64)
    Bf = inputs.bf16_bits_to_f32(Bt).astype(np.float64)
    C = oracle.matmul_bf16(A, Bt)
    assert np.allclose(C, Af @ Bf.T, rtol=0, atol=1e-12)
    r = inputs.uniform_f32(3, N).astype(np.float64)
    assert np.allclose(C @ r, Af @ (Bf.T @ r), atol=1e-9)
    rows = np.array([0, 5, 39, 17], np.int64)
    cols = np.array([0, 55, 3, 28], np.int64)
    s, sa = oracle.matmul_bf16_sampled(A, Bt, rows, cols)
    assert np.allclose(s, C[rows, cols], atol=1e-12)
    assert np.allclose(sa, np.abs(Af[rows] * Bf[cols]).sum(1))


def test_bf16_rounding_is_rne():
    x = np.array([1.0, 1.0 + 2**-8, 1.0 + 3 * 2**-9, -2.5, 3.0e38], np.float32)
    b = inputs.f32_to_bf16_bits(x)
    back = inputs.bf16_bits_to_f32(b)
    assert back[0] == 1.0 and back[1] == 1.0  # tie -> even
    assert back[2] == 1.0 + 2**-7  # above half -> up
    assert back[3] == -2.5


# ---------------------------------------------------------------- BitonicSort (R-BIT1)


def test_sort_vs_library_and_invariants():
    for bits in (32, 8, 1):
        k = inputs.bitonic_keys(21, 1 << 14, bits=bits)
        s = oracle.sort_u32(k)
        assert np.array_equal(s, np.sort(k))                      # library routine
        assert np.all(s[1:] >= s[:-1])                            # sorted
        assert np.array_equal(np.unique(s, return_counts=True)[1],  # same multiset
                              np.unique(k, return_counts=True)[1])
    assert np.array_equal(oracle.sort_u32(np.arange(1024, dtype=np.uint32)[::-1].copy()),
                          np.arange(1024, dtype=np.uint32))
    assert np.array_equal(oracle.sort_u32(np.array([7], np.uint32)), np.array([7], np.uint32))
    assert np.array_equal(oracle.sort_u32(np.full(64, 0xFFFFFFFF, np.uint32)), np.full(64, 0xFFFFFFFF, np.uint32))


def test_sort_brute_force_permutations():
    base = [0, 1, 1, 2, 3, 5, 8, 0xFFFFFFFF]
    for perm in itertools.islice(itertools.permutations(base), 0, 40320, 17):
        assert list(oracle.sort_u32(np.array(perm, np.uint32))) == sorted(base)


# ---------------------------------------------------------------- DwtHaar1D (R-DWT1/2)


def _haar_basis(N):
    """Rows = the orthonormal Haar functions in the R-DWT1 output layout."""
    L = N.bit_length() - 1
    H = np.zeros((N, N))
    H[0, :] = 2.0 ** (-L / 2)
    for k in range(1, L + 1):
        w = 1 << k
        for j in range(N >> k):
            row = (N >> k) + j
            H[row, j * w: j * w + w // 2] = 2.0 ** (-k / 2)
            H[row, j * w + w // 2: (j + 1) * w] = -(2.0 ** (-k / 2))
    return H


def test_dwt_haar_basis_closed_form():
    for N in (1, 2, 4, 8, 64, 256):
        x = inputs.dwt_x(3, N)
        y = oracle.dwthaar1d_f64(x)
        assert np.allclose(y, _haar_basis(N) @ x.astype(np.float64), rtol=0, atol=1e-12), N


def test_dwt_parseval_constant_and_inverse():
    N = 1 << 12
    x = inputs.dwt_x(4, N)
    y = oracle.dwthaar1d_f64(x)
    assert abs(np.dot(y, y) - np.dot(x.astype(np.float64), x)) < 1e-9 * np.dot(x.astype(np.float64), x)
    c = oracle.dwthaar1d_f64(np.full(N, 0.5, np.float32))
    assert abs(c[0] - 0.5 * math.sqrt(N)) < 1e-12 and np.all(np.abs(c[1:]) < 1e-12)
    # inverse, written independently: coarse to fine, c_{2i} = (a+d)/sqrt2, c_{2i+1} = (a-d)/sqrt2
    a = y[:1].copy()
    n = 1
    while n < N:
        d = y[n:2 * n]
        nxt = np.empty(2 * n)
        nxt[0::2] = (a + d) / math.sqrt(2.0)
        nxt[1::2] = (a - d) / math.sqrt(2.0)
        a, n = nxt, 2 * n
    assert np.allclose(a, x.astype(np.float64), rtol=0, atol=1e-12)


def test_dwt_f32dag_within_rounding_bound():
    N = 1 << 14
    x = inputs.dwt_x(5, N)
    y64 = oracle.dwthaar1d_f64(x)
    y32 = oracle.dwthaar1d_f32dag(x).astype(np.float64)
    # every coefficient is a signed sum over its support scaled by 2^{-k/2}; each
    # level adds <= 2 roundings: |err| <= 2 L u * (same transform of |x| with + only)
    L = N.bit_length() - 1
    absb = oracle.dwthaar1d_f64(np.abs(x))  # a-path of |x| bounds |a|; details bounded by the same a
    bound = np.empty(N)
    bound[0] = absb[0]
    for k in range(1, L + 1):
        lo, hi = N >> k, N >> (k - 1)
        # level-k |coefficient| <= 2^{-k/2} * sum |x| over 2^k samples = level-k a of |x|
        ax = np.abs(x.astype(np.float64)).reshape(-1, 1 << k).sum(axis=1) * 2.0 ** (-k / 2)
        bound[lo:hi] = ax
    assert np.all(np.abs(y32 - y64) <= 2 * L * 2.0 ** -24 * bound + 1e-30)


# ---------------------------------------------------------------- BinomialOption (R-BO1/2)


def _crr_closed_form(S, K, T, R, V, N, call=True):
    """Independent form: discounted binomial expectation of the payoff."""
    dt = T / N
    u = math.exp(V * math.sqrt(dt))
    d = 1 / u
    p = (math.exp(R * dt) - d) / (u - d)
    tot = 0.0
    for k in range(N + 1):
        ST = S * u ** (2 * k - N)
        pay = max(ST - K, 0.0) if call else max(K - ST, 0.0)
        if pay > 0:
            lw = (math.lgamma(N + 1) - math.lgamma(k + 1) - math.lgamma(N - k + 1)
                  + k * math.log(p) + (N - k) * math.log1p(-p))
            tot += math.exp(lw) * pay
    return math.exp(-R * T) * tot


def test_bo_lattice_vs_closed_form_sum():
    for r in (0.0, 0.13, 0.5, 0.77, 1.0):
        S, K, T = oracle.bo_params(r)
        for call in (True, False):
            a = oracle.crr_price(S, K, T, oracle.BO_R, oracle.BO_V, oracle.BO_STEPS, call)
            b = _crr_closed_form(S, K, T, oracle.BO_R, oracle.BO_V, oracle.BO_STEPS, call)
            assert abs(a - b) <= 1e-9 * max(1.0, abs(b)), (r, call, a, b)
    # N = 1 by hand
    S, K, T, R, V = 20.0, 21.0, 1.0, 0.05, 0.3
    u = math.exp(V); d = 1 / u; p = (math.exp(R) - d) / (u - d)
    hand = math.exp(-R) * (p * max(S * u - K, 0) + (1 - p) * max(S * d - K, 0))
    assert abs(oracle.crr_price(S, K, T, R, V, 1, True) - hand) < 1e-12


def test_bo_put_call_parity_bounds_and_bs_limit():
    for r in np.linspace(0, 1, 11):
        S, K, T = oracle.bo_params(r)
        C = oracle.crr_price(S, K, T, oracle.BO_R, oracle.BO_V, oracle.BO_STEPS, True)
        P = oracle.crr_price(S, K, T, oracle.BO_R, oracle.BO_V, oracle.BO_STEPS, False)
        disc = K * math.exp(-oracle.BO_R * T)
        assert abs((C - P) - (S - disc)) < 1e-9 * S          # exact on the lattice
        assert max(0.0, S - disc) - 1e-12 <= C <= S
        bs_c, _ = oracle.bs_price(S, K, T, oracle.BO_R, oracle.BO_V)
        assert abs(C - bs_c) < 5e-3 * S                       # CRR -> Black-Scholes, O(1/N)
    # the error shrinks with N (first-order convergence, at-the-money)
    e1 = abs(oracle.crr_price(100, 100, 1, 0.05, 0.2, 64, True) - 10.450575619322287)
    e2 = abs(oracle.crr_price(100, 100, 1, 0.05, 0.2, 1024, True) - 10.450575619322287)
    assert e2 < e1 / 4


def test_bo_workload_mapping():
    assert oracle.bo_params(0.0) == (5.0, 1.0, 0.25)
    assert oracle.bo_params(1.0) == (30.0, 100.0, 10.0)
    r = inputs.binomial_r(7, 64)
    v = oracle.binomialoption(r)
    for i in (0, 17, 63):
        S, K, T = oracle.bo_params(float(r[i]))
        assert v[i] == oracle.crr_price(S, K, T, oracle.BO_R, oracle.BO_V, oracle.BO_STEPS, True)
