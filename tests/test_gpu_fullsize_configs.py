"""Full-size parity (-m gpu) for the BASELINE.json configs other than
configs[1] (tests/test_gpu_fullsize.py), at their full sizes and in the launch
configuration bench.py times (workloads.config_jobs): the unprotected kernel
against the oracle on sampled outputs the oracle computes one by one, or via
properties that hold at any size; every BASELINE.json RMT variant (plus the
cluster form) bitwise equal to the unprotected output with zero false alarms.

  configs[2] suite28: BinarySearch N=2^28 Q=2^26, FWT / PrefixSum / Reduction
             2^28, Transpose / Sobel 16384^2
  configs[3] fwdct  : FloydWarshall 4096 nodes, DCT 8192^2
  configs[4] bs30 / mm16k: BlackScholes 2^30 options, MatrixMultiplication
             16384^3 (integer-valued inputs: the exactness pin; random: Freivalds
             + sampled fp64 dots)
"""
import numpy as np
import pytest
import torch

import oracle
from paper_conf_isca_waddenlgss14_b200 import inputs, rmt, workloads

pytestmark = pytest.mark.gpu

VARIANTS = ("intra_smem", "intra_reg", "inter_group", "inter_cluster")


def _run(j, variant, bufs):
    outs = [i for i, h in enumerate(j.host_in) if h is None]
    if j.kernel == "floydwarshall":  # D is in/out: restart from W
        bufs[0].copy_(torch.from_numpy(j.host_in[0].view(np.int32).reshape(-1)).cuda())
    for i in outs:
        bufs[i].fill_(-1)
    err = torch.zeros(1, dtype=torch.int64, device="cuda")
    ws = rmt.make_workspace(j.kernel, variant, j.n, j.dims)
    rmt.launch(j.kernel, variant, bufs, j.n, err, dims=j.dims, workspace=ws)
    torch.cuda.synchronize()
    del ws
    res = [bufs[0].cpu().numpy().copy()] if j.kernel == "floydwarshall" else []
    res += [bufs[i].cpu().numpy().copy() for i in outs]
    return int(err.item()), res


def _variants_identical(j, bufs, ref):
    for v in VARIANTS:
        err, outs = _run(j, v, bufs)
        assert err == 0, f"{j.kernel}/{v}: {err} false alarms at full size"
        for a, b in zip(outs, ref):
            assert np.array_equal(a, b), f"{j.kernel}/{v} differs from none at full size"


def _release(j):
    j.dev = None
    torch.cuda.empty_cache()


# ---------------------------------------------------------------- configs[2]
SUITE28 = None


def _suite28():
    global SUITE28
    if SUITE28 is None:
        SUITE28 = {j.kernel: j for j in workloads.config_jobs("suite28")}
    return SUITE28


def _check_suite28(j, outs):
    rng = np.random.default_rng(1)
    if j.kernel == "binarysearch":
        A, q = j.host_in[0], j.host_in[1]
        s = rng.integers(0, q.size, 1 << 14)
        assert np.array_equal(outs[0].view(np.uint32)[s], oracle.binarysearch(A, q[s]))
    elif j.kernel == "fwt":
        # R-FWT2: the stage order fixes the fp32 result; full output vs the fp32-DAG oracle
        assert np.array_equal(outs[0].view(np.uint32), oracle.fwt_f32dag(j.host_in[0]).view(np.uint32))
    elif j.kernel == "prefixsum":
        assert np.array_equal(outs[0].view(np.uint32), oracle.prefixsum_u32(j.host_in[0]))
    elif j.kernel == "reduction":
        assert int(outs[0].view(np.uint64)[0]) == oracle.reduction_u32(j.host_in[0])
    elif j.kernel == "transpose":
        H, W = j.dims
        s = rng.integers(0, H, 128)
        got = outs[0].view(np.uint32).reshape(W, H)
        assert np.array_equal(got[:, s], oracle.transpose_u32(j.host_in[0].reshape(H, W)[s]))
    elif j.kernel == "sobel":
        H, W = j.dims
        I = j.host_in[0].reshape(H, W).view(np.uint8).reshape(H, W, 4)
        got = outs[0].view(np.uint32).reshape(H, W)
        for r in list(rng.integers(1, H - 1, 24)) + [0, 1, H - 2, H - 1]:
            lo, hi = max(0, r - 1), min(H, r + 2)
            band = oracle.sobel(np.ascontiguousarray(I[lo:hi])).view(np.uint32).reshape(hi - lo, W)
            if 0 < r < H - 1:
                assert np.array_equal(got[r], band[r - lo])
            else:
                assert not got[r].any()


@pytest.mark.parametrize("kernel", ["binarysearch", "fwt", "prefixsum", "reduction", "transpose", "sobel"])
def test_suite28_fullsize(kernel):
    j = _suite28()[kernel]
    bufs = j.device_buffers()
    err, ref = _run(j, "none", bufs)
    assert err == 0
    _check_suite28(j, ref)
    _variants_identical(j, bufs, ref)
    _release(j)


def test_prefixsum_f32_fullsize():
    """The fp32 PrefixSum (fixed association, dims[2] bit 1) at the suite size
    2^26, inclusive and exclusive: within 1e-5 of the fp64 definition scaled by
    sum |x_j|, every variant bitwise equal to none."""
    n = 1 << 26
    x = inputs.prefixsum_f32(4, n)
    xd = torch.from_numpy(x).cuda()
    y = torch.empty(n, dtype=torch.float32, device="cuda")
    for excl in (False, True):
        dims = (0, 0, 2 | (1 if excl else 0))
        ref = None
        for v in ["none", *VARIANTS]:
            y.fill_(float("nan"))
            err = torch.zeros(1, dtype=torch.int64, device="cuda")
            ws = rmt.make_workspace("prefixsum", v, n, dims)
            rmt.launch("prefixsum", v, [xd, y], n, err, dims=dims, workspace=ws)
            torch.cuda.synchronize()
            got = y.cpu().numpy().view(np.uint32).copy()
            assert int(err.item()) == 0, f"prefixsum f32/{v}: false alarms"
            if ref is None:
                ref = got
                yo, bo = oracle.prefixsum_f64(x, exclusive=excl)
                d = np.abs(got.view(np.float32).astype(np.float64) - yo)
                assert np.all(d <= 1e-5 * bo + 1e-30), float(np.max(d / (bo + 1e-30)))
            else:
                assert np.array_equal(got, ref), f"prefixsum f32/{v} differs from none"
    del xd, y
    torch.cuda.empty_cache()


# ---------------------------------------------------------------- configs[3]
def test_floydwarshall_4096_fullsize():
    j = workloads.job_floydwarshall(4096)
    n = j.n
    bufs = j.device_buffers()
    err, ref = _run(j, "none", bufs)
    assert err == 0
    D = ref[0].view(np.uint32).reshape(n, n)
    P = ref[1].view(np.uint32).reshape(n, n)
    Wm = j.host_in[0].reshape(n, n)
    rng = np.random.default_rng(2)
    # D rows against Dijkstra (an independent algorithm), P by the path invariant
    for src in list(rng.integers(0, n, 6)) + [0, n - 1]:
        assert np.array_equal(D[src], oracle.dijkstra_row(Wm, int(src)))
        p = P[src].astype(np.int64)
        direct = p == src
        assert np.array_equal(D[src][direct], Wm[src][direct])
        via = ~direct
        cols = np.nonzero(via)[0]
        assert np.array_equal(D[src][cols].astype(np.int64), D[src, p[cols]].astype(np.int64) + D[p[cols], cols])
    assert not np.diag(D).any()
    _variants_identical(j, bufs, ref)
    _release(j)


def test_dct_8192_fullsize():
    j = workloads.job_dct(8192, 8192)
    H, W = j.dims
    bufs = j.device_buffers()
    err, ref = _run(j, "none", bufs)
    assert err == 0
    Y = ref[0].view(np.float32).reshape(H, W).astype(np.float64)
    X = j.host_in[0].reshape(H, W)
    rng = np.random.default_rng(3)
    for s in list(rng.integers(0, H // 8, 16)) + [0, H // 8 - 1]:
        band = np.ascontiguousarray(X[8 * s:8 * s + 8])
        yr = oracle.dct8x8(band)
        bound = oracle.dct8x8_absbound(band)
        # R-DCT3: componentwise 1e-5 of the condition bound
        assert np.all(np.abs(Y[8 * s:8 * s + 8] - yr) <= 1e-5 * bound + 1e-30)
    _variants_identical(j, bufs, ref)
    _release(j)


# ---------------------------------------------------------------- configs[4]
def test_blackscholes_2p30_fullsize():
    j = workloads.job_blackscholes(1 << 30)
    bufs = j.device_buffers()
    err, ref = _run(j, "none", bufs)
    assert err == 0
    r = j.host_in[0]
    call = ref[0].view(np.float32)
    put = ref[1].view(np.float32)
    # put-call parity on every option (a closed form, independent of the CND)
    for lo in range(0, r.size, 1 << 26):
        rr = r[lo:lo + (1 << 26)].astype(np.float64)
        S = 10 * rr + 100 * (1 - rr)
        T = rr + 10 * (1 - rr)
        R = 0.01 * rr + 0.05 * (1 - rr)
        c = call[lo:lo + (1 << 26)].astype(np.float64)
        p = put[lo:lo + (1 << 26)].astype(np.float64)
        assert np.all(np.abs(c - p - (S - S * np.exp(-R * T))) <= 1e-4 * S)
    rng = np.random.default_rng(4)
    s = rng.integers(0, r.size, 1 << 16)
    cr, pr = oracle.blackscholes(r[s])
    S = 10 * r[s].astype(np.float64) + 100 * (1 - r[s].astype(np.float64))
    for got, want in ((call[s], cr), (put[s], pr)):
        assert np.all(np.abs(got - want) <= 1e-4 * np.maximum(np.abs(want), 1e-2 * S))
    _variants_identical(j, bufs, ref)
    _release(j)


@pytest.mark.parametrize("integer", [True, False])
def test_matmul_16384_fullsize(integer):
    M = N = K = 16384
    if integer:
        A = inputs.matmul_bf16_int(10, M, K, stream=20)
        Bt = inputs.matmul_bf16_int(10, N, K, stream=21)
        j = workloads.Job("matmul", M * N, (M, N, K), [A, Bt, None], [(2, 4 * M * N)], alg_bytes=0, unit="C")
    else:
        j = workloads.job_matmul(M, N, K)
        A, Bt = j.host_in[0], j.host_in[1]
    bufs = j.device_buffers()
    err, ref = _run(j, "none", bufs)
    assert err == 0
    C = ref[0].view(np.float32).reshape(M, N)
    Af = inputs.bf16_bits_to_f32(A.reshape(M, K)).astype(np.float64)
    Bf = inputs.bf16_bits_to_f32(Bt.reshape(N, K)).astype(np.float64)
    rng = np.random.default_rng(5)
    x = rng.standard_normal(N)
    # Freivalds: C x == A (B^T x) (O(n^2), fp64)
    lhs = C.astype(np.float64) @ x
    rhs = Af @ (Bf.T @ x)
    if integer:
        xi = rng.integers(-3, 4, N).astype(np.float64)  # exact in fp64 (|terms| < 2^53)
        assert np.array_equal(C.astype(np.float64) @ xi, Af @ (Bf.T @ xi))
    # R-MM2: normwise 1e-5 (BASELINE.json).  R-MM4: the tensor pipe's own fp32
    # accumulation is not round-to-nearest (1.9e-5 at K = 16384 in one TMEM
    # accumulator); the kernel accumulates K in chunks of 1024 and adds them RN
    rel = np.linalg.norm(lhs - rhs) / np.linalg.norm(rhs)
    print(f"matmul 16384^3 normwise error (Freivalds projection): {rel:.3e}")
    assert rel <= 1e-5
    rows = rng.integers(0, M, 4096)
    cols = rng.integers(0, N, 4096)
    want, absw = oracle.matmul_bf16_sampled(A.reshape(M, K), Bt.reshape(N, K), rows, cols)
    got = C[rows, cols].astype(np.float64)
    if integer:
        assert np.array_equal(got, want)  # exactness pin at full size
    else:
        assert np.all(np.abs(got - want) <= K * 2.0 ** -23 * absw + 1e-30)
    _variants_identical(j, bufs, ref)
    _release(j)
