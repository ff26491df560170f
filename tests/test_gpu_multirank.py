"""Sharded == single GPU, through librmt (-m gpu).

Two ranks share the one GPU of the test box (gloo process group: NCCL refuses
two ranks on one device, and gloo stages the few collectives through the host;
the NCCL path uses the same parallel.py functions on device tensors).  Every
shardable kernel runs sharded through parallel.py + librmt under the
unprotected and the three BASELINE.json RMT variants, the shards are gathered,
and rank 0 checks them bitwise against the same kernel run on the whole
problem in one process -- FWT across shards (local transform + a cross-shard
butterfly stage), PrefixSum with the device-side carry, Reduction's all-reduce,
Sobel with halo rows, and the independent row/element shards.
"""
import os
import socket
import traceback

import numpy as np
import pytest
import torch

pytestmark = pytest.mark.gpu

WS = 2
VARIANTS = ("none", "intra_smem", "intra_reg", "inter_group")


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _run(rmt, kernel, variant, bufs, n, dims=()):
    err = torch.zeros(1, dtype=torch.int64, device="cuda")
    ws = rmt.make_workspace(kernel, variant, n, dims)
    rmt.launch(kernel, variant, bufs, n, err, dims=dims, workspace=ws)
    torch.cuda.synchronize()
    return int(err.item())


def _dev(a):
    a = np.ascontiguousarray(a)
    view = {np.dtype(np.uint32): np.int32, np.dtype(np.uint16): np.int16}.get(a.dtype, a.dtype)
    return torch.from_numpy(a.view(view).copy()).cuda()


def _zeros(nwords):
    return torch.full((max(nwords, 4),), -1, dtype=torch.int32, device="cuda")[:nwords]


def _shards(rank):
    """(kernel, sharded runner, whole-problem runner) per shardable kernel; each
    runner returns (err, numpy result) for one variant."""
    import torch.distributed as dist

    from paper_conf_isca_waddenlgss14_b200 import inputs, parallel, rmt

    cases = {}

    # BlackScholes: contiguous option ranges (strong: 2^20 split over the ranks)
    n = 1 << 20
    off, cnt = parallel.strong_range(n, WS, rank, align=4)

    def bs_shard(v):
        r = _dev(inputs.blackscholes_r(1, cnt, off))
        c, p = _zeros(cnt), _zeros(cnt)
        return _run(rmt, "blackscholes", v, [r, c, p], cnt, (0,)), np.concatenate([c.cpu().numpy(), p.cpu().numpy()])

    def bs_full(v):
        r = _dev(inputs.blackscholes_r(1, n))
        c, p = _zeros(n), _zeros(n)
        e = _run(rmt, "blackscholes", v, [r, c, p], n, (0,))
        return e, [np.concatenate([c.cpu().numpy()[o:o + k], p.cpu().numpy()[o:o + k]])
                   for o, k in (parallel.strong_range(n, WS, q, 4) for q in range(WS))]
    cases["blackscholes"] = (bs_shard, bs_full)

    # BinarySearch: queries sharded, A replicated
    N, Q = 1 << 20, 1 << 18
    A, qall = inputs.binarysearch_inputs(6, N, Q)
    qo, qc = parallel.strong_range(Q, WS, rank, align=4)

    def bins_shard(v):
        out = _zeros(qc)
        return _run(rmt, "binarysearch", v, [_dev(A), _dev(qall[qo:qo + qc]), out], qc, (N, qc)), out.cpu().numpy()

    def bins_full(v):
        out = _zeros(Q)
        e = _run(rmt, "binarysearch", v, [_dev(A), _dev(qall), out], Q, (N, Q))
        return e, [out.cpu().numpy()[o:o + k] for o, k in (parallel.strong_range(Q, WS, q, 4) for q in range(WS))]
    cases["binarysearch"] = (bins_shard, bins_full)

    # FWT: local transform of N/G + log2 G cross-shard stages
    NF = 1 << 20
    nl = NF // WS

    def fwt_shard(v):
        x = _dev(inputs.fwt_x(5, nl, rank * nl))
        y, recv, tmp = (torch.empty(nl, dtype=torch.float32, device="cuda") for _ in range(3))
        err = torch.zeros(1, dtype=torch.int64, device="cuda")
        parallel.global_fwt(x, y, recv, tmp, err, rmt, v, workspace=rmt.make_workspace("fwt", v, nl),
                            ws_comb=rmt.make_workspace("fwt", v, nl, (1, 0)))
        torch.cuda.synchronize()
        return int(err.item()), y.cpu().numpy().view(np.uint32)

    def fwt_full(v):
        x = _dev(inputs.fwt_x(5, NF))
        y = torch.empty(NF, dtype=torch.float32, device="cuda")
        e = _run(rmt, "fwt", v, [x, y], NF, (0,))
        yy = y.cpu().numpy().view(np.uint32)
        return e, [yy[q * nl:(q + 1) * nl] for q in range(WS)]
    cases["fwt"] = (fwt_shard, fwt_full)

    # the fused FWT: the combine kernel reads the partner's shard through CUDA IPC
    # (peer-to-peer over NVLink on a multi-GPU box; shared memory of one GPU here)
    peer = parallel.PeerFWT(nl, rmt)

    def fwt_p2p_shard(v):
        x = _dev(inputs.fwt_x(5, nl, rank * nl))
        err = torch.zeros(1, dtype=torch.int64, device="cuda")
        y, _ = peer.run(x, err, v, workspace=rmt.make_workspace("fwt", v, nl),
                        ws_comb=rmt.make_workspace("fwt", v, nl, (1, 0)))
        torch.cuda.synchronize()
        return int(err.item()), y.cpu().numpy().view(np.uint32)
    cases["fwt_p2p"] = (fwt_p2p_shard, fwt_full)

    # PrefixSum: device all-gather of the shard totals -> device carry
    npl = (1 << 19) + 1028

    def ps_shard(v):
        x = _dev(inputs.prefixsum_x(4, npl, rank * npl))
        y = _zeros(npl)
        s_tmp = torch.zeros(2, dtype=torch.int32, device="cuda")
        totals = torch.zeros(WS, dtype=torch.int64, device="cuda")
        err = torch.zeros(1, dtype=torch.int64, device="cuda")
        parallel.global_prefixsum(x, y, s_tmp, totals, err, rmt, v, ws_red=rmt.make_workspace("reduction", v, npl),
                                  ws_ps=rmt.make_workspace("prefixsum", v, npl))
        torch.cuda.synchronize()
        return int(err.item()), y.cpu().numpy().view(np.uint32)

    def ps_full(v):
        x = _dev(inputs.prefixsum_x(4, npl * WS))
        y = _zeros(npl * WS)
        e = _run(rmt, "prefixsum", v, [x, y], npl * WS, (0,))
        yy = y.cpu().numpy().view(np.uint32)
        return e, [yy[q * npl:(q + 1) * npl] for q in range(WS)]
    cases["prefixsum"] = (ps_shard, ps_full)

    # Reduction: all-reduce of the shard sums
    nr = (1 << 20) + 3

    def red_shard(v):
        x = _dev(inputs.reduction_x(2, nr, rank * nr))
        s = torch.zeros(1, dtype=torch.int64, device="cuda")
        err = torch.zeros(1, dtype=torch.int64, device="cuda")
        parallel.global_reduction(x, s, err, rmt, v, workspace=rmt.make_workspace("reduction", v, nr))
        torch.cuda.synchronize()
        return int(err.item()), s.cpu().numpy().view(np.uint64)

    def red_full(v):
        x = _dev(inputs.reduction_x(2, nr * WS))
        s = torch.zeros(1, dtype=torch.int64, device="cuda")
        e = _run(rmt, "reduction", v, [x, s], nr * WS)
        return e, [s.cpu().numpy().view(np.uint64)] * WS
    cases["reduction"] = (red_shard, red_full)

    # Transpose: row block of A -> column block of B
    H, W = 512, 768
    h0, hc = parallel.strong_range(H, WS, rank, align=4)

    def tr_shard(v):
        a = _dev(inputs.transpose_a(3, hc, W, h0).view(np.uint32))
        b = _zeros(hc * W)
        return _run(rmt, "transpose", v, [a, b], hc * W, (hc, W)), b.cpu().numpy().view(np.uint32).reshape(W, hc)

    def tr_full(v):
        a = _dev(inputs.transpose_a(3, H, W).view(np.uint32))
        b = _zeros(H * W)
        e = _run(rmt, "transpose", v, [a, b], H * W, (H, W))
        bb = b.cpu().numpy().view(np.uint32).reshape(W, H)
        return e, [np.ascontiguousarray(bb[:, o:o + k]) for o, k in (parallel.strong_range(H, WS, q, 4) for q in range(WS))]
    cases["transpose"] = (tr_shard, tr_full)

    # Sobel: row blocks with one halo row above / below
    HS, WSb = 256, 512
    s0, sc = parallel.strong_range(HS, WS, rank)
    lo, hi = parallel.sobel_halo_rows(HS, s0, s0 + sc)

    def sob_shard(v):
        img = _dev(inputs.sobel_image(7, hi - lo, WSb, lo).view(np.uint32).reshape(-1))
        o = _zeros((hi - lo) * WSb)
        e = _run(rmt, "sobel", v, [img, o], (hi - lo) * WSb, (hi - lo, WSb))
        return e, o.cpu().numpy().view(np.uint32).reshape(hi - lo, WSb)[s0 - lo:s0 - lo + sc]

    def sob_full(v):
        img = _dev(inputs.sobel_image(7, HS, WSb).view(np.uint32).reshape(-1))
        o = _zeros(HS * WSb)
        e = _run(rmt, "sobel", v, [img, o], HS * WSb, (HS, WSb))
        oo = o.cpu().numpy().view(np.uint32).reshape(HS, WSb)
        return e, [oo[o_:o_ + k] for o_, k in (parallel.strong_range(HS, WS, q) for q in range(WS))]
    cases["sobel"] = (sob_shard, sob_full)

    # DCT: row blocks of 8-row multiples
    HD, WD = 256, 512
    d0, dc = parallel.strong_range(HD, WS, rank, align=8)

    def dct_shard(v):
        x = _dev(inputs.dct_x(9, dc, WD, d0))
        y = _zeros(dc * WD)
        return _run(rmt, "dct", v, [x, y], dc * WD, (dc, WD)), y.cpu().numpy().view(np.uint32)

    def dct_full(v):
        x = _dev(inputs.dct_x(9, HD, WD))
        y = _zeros(HD * WD)
        e = _run(rmt, "dct", v, [x, y], HD * WD, (HD, WD))
        yy = y.cpu().numpy().view(np.uint32)
        return e, [yy[o * WD:(o + k) * WD] for o, k in (parallel.strong_range(HD, WS, q, 8) for q in range(WS))]
    cases["dct"] = (dct_shard, dct_full)

    # MatrixMultiplication: rows of A and C, B replicated
    M, NN, K = 512, 256, 512
    m0, mc = parallel.strong_range(M, WS, rank, align=128)

    def mm_shard(v):
        a = _dev(inputs.matmul_bf16_normal(10, mc, K, stream=22, row_offset=m0))
        b = _dev(inputs.matmul_bf16_normal(10, NN, K, stream=24))
        c = _zeros(mc * NN)
        return _run(rmt, "matmul", v, [a, b, c], mc * NN, (mc, NN, K)), c.cpu().numpy().view(np.uint32)

    def mm_full(v):
        a = _dev(inputs.matmul_bf16_normal(10, M, K, stream=22))
        b = _dev(inputs.matmul_bf16_normal(10, NN, K, stream=24))
        c = _zeros(M * NN)
        e = _run(rmt, "matmul", v, [a, b, c], M * NN, (M, NN, K))
        cc = c.cpu().numpy().view(np.uint32)
        return e, [cc[o * NN:(o + k) * NN] for o, k in (parallel.strong_range(M, WS, q, 128) for q in range(WS))]
    cases["matmul"] = (mm_shard, mm_full)
    return cases


def _worker(rank, port, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    try:
        torch.cuda.set_device(0)
        dist.init_process_group("gloo", rank=rank, world_size=WS)
        cases = _shards(rank)
        failures = []
        for kernel, (shard, full) in cases.items():
            for v in VARIANTS:
                e, mine = shard(v)
                got = [None] * WS
                dist.all_gather_object(got, (e, mine))
                if rank == 0:
                    ef, ref = full(v)
                    if ef != 0 or any(g[0] != 0 for g in got):
                        failures.append(f"{kernel}/{v}: err {[g[0] for g in got]} full {ef}")
                    for r in range(WS):
                        if not np.array_equal(np.asarray(got[r][1]).reshape(-1), np.asarray(ref[r]).reshape(-1)):
                            failures.append(f"{kernel}/{v}: rank {r} shard != single-GPU result")
        q.put((rank, failures))
        dist.barrier()
        dist.destroy_process_group()
    except Exception:
        q.put((rank, [traceback.format_exc()]))


def test_sharded_equals_single_gpu():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, port, q)) for r in range(WS)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=600) for _ in range(WS))
    for p in procs:
        p.join(60)
    assert res[1] == [], res[1]
    assert res[0] == [], "\n".join(res[0])
