"""Multi-process (gloo, world_size 2, CPU) tests of the multi-GPU host logic in
paper_conf_isca_waddenlgss14_b200/parallel.py: shard generation, the PrefixSum
carry-in all-gather, the Reduction and error-counter all-reduces.  Kernels need
a GPU, so each rank's local kernel result is stood in by the oracle; what is
tested is that the collectives turn per-shard results into the global ones."""
import os
import socket

import numpy as np
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
from paper_conf_isca_waddenlgss14_b200 import inputs, parallel

N_PER = 5003  # deliberately not a multiple of anything


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


class _OracleRmt:
    """Stand-in for the rmt binding on CPU tensors (no GPU here): the oracle
    (and, for the FWT cross-shard stage, its definition written out in fp32)
    in place of each kernel, so the host logic of parallel.py -- partner
    pairing, stage order, upper/lower roles, the device-tensor all-gather of
    the totals and the carry -- is what is tested."""

    def launch(self, kernel, variant, bufs, n, err, dims=(), workspace=None, stream=None):
        if kernel == "fwt" and dims[0] == 0:
            bufs[1].copy_(torch.from_numpy(oracle.fwt_f32dag(bufs[0].numpy())))
        elif kernel == "fwt":
            x, p = bufs[0].numpy(), bufs[2].numpy()
            bufs[1].copy_(torch.from_numpy((p - x) if dims[1] else (x + p)))  # fp32 elementwise
        elif kernel == "reduction":
            bufs[1].view(torch.int64)[0] = oracle.reduction_u32(bufs[0].numpy().view(np.uint32))
        elif kernel == "prefixsum":
            carry = int(dims[0]) if dims else 0
            if len(bufs) > 2:
                carry += int(bufs[2][: dims[1]].sum())
            y = (oracle.prefixsum_u32(bufs[0].numpy().view(np.uint32)).astype(np.uint64) + carry) % 2**32
            bufs[1].copy_(torch.from_numpy(y.astype(np.uint32).view(np.int32)))
        return 1


def _worker_global(rank, ws, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=ws)
    try:
        fake = _OracleRmt()
        err = torch.zeros(1, dtype=torch.int64)
        # FWT across ws shards == the single-GPU fp32 DAG (bitwise)
        nl = 1 << 12
        x = torch.from_numpy(inputs.fwt_x(5, nl, rank * nl))
        y, recv, tmp = (torch.empty(nl, dtype=torch.float32) for _ in range(3))
        parallel.global_fwt(x, y, recv, tmp, err, fake)
        ref = oracle.fwt_f32dag(inputs.fwt_x(5, nl * ws))[rank * nl:(rank + 1) * nl]
        assert np.array_equal(y.numpy().view(np.uint32), ref.view(np.uint32)), "global FWT shard differs"
        # PrefixSum with the all-gathered totals and the carry
        npl = 1000 + 7 * rank
        sizes = [1000 + 7 * r for r in range(ws)]
        off = sum(sizes[:rank])
        xg = inputs.prefixsum_x(4, sum(sizes), 0)
        xs = torch.from_numpy(xg[off:off + npl].view(np.int32).copy())
        ys = torch.empty(npl, dtype=torch.int32)
        totals = torch.zeros(ws, dtype=torch.int64)
        parallel.global_prefixsum(xs, ys, torch.zeros(2, dtype=torch.int32), totals, err, fake)
        assert np.array_equal(ys.numpy().view(np.uint32), oracle.prefixsum_u32(xg)[off:off + npl])
        # strong-scaling shards tile the global range
        parts = [parallel.strong_range(1 << 20, ws, r, 4) for r in range(ws)]
        assert parts[0][0] == 0 and sum(c for _, c in parts) == 1 << 20
        assert all(parts[r][0] + parts[r][1] == parts[r + 1][0] for r in range(ws - 1))
        q.put((rank, "ok"))
    except Exception as ex:
        q.put((rank, repr(ex)))
    finally:
        dist.destroy_process_group()


def _spawn(target, ws):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=target, args=(r, ws, port, q)) for r in range(ws)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=120) for _ in range(ws))
    for p in procs:
        p.join(60)
    return res


def test_global_fwt_and_prefixsum_host_logic_gloo():
    for ws in (2, 4):
        res = _spawn(_worker_global, ws)
        assert all(v == "ok" for v in res.values()), res


def _worker(rank, ws, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=ws)
    try:
        off, cnt = parallel.shard_range(N_PER, rank)
        x = inputs.prefixsum_x(4, cnt, off)               # this rank's shard, generated locally
        xg = inputs.prefixsum_x(4, N_PER * ws, 0)         # the 1-GPU input
        assert np.array_equal(x, xg[off:off + cnt])
        # PrefixSum: local scan + carry-in from the all-gather == global scan slice
        local_total = oracle.reduction_u32(x)
        carry = parallel.exclusive_carry(local_total)
        y = (oracle.prefixsum_u32(x).astype(np.uint64) + carry) % 2**32
        assert np.array_equal(y.astype(np.uint32), oracle.prefixsum_u32(xg)[off:off + cnt])
        # Reduction: all-reduce of the local u64 sums == global sum
        r = inputs.reduction_x(2, cnt, off)
        t = torch.tensor([oracle.reduction_u32(r)], dtype=torch.int64)
        parallel.allreduce_sum_(t)
        assert int(t.item()) == oracle.reduction_u32(inputs.reduction_x(2, N_PER * ws, 0))
        # error counters: per-rank counts sum
        e = torch.tensor([rank + 1], dtype=torch.int64)
        parallel.allreduce_sum_(e)
        assert int(e.item()) == ws * (ws + 1) // 2
        q.put((rank, "ok"))
    except Exception as ex:  # surface the failure to the parent
        q.put((rank, repr(ex)))
    finally:
        dist.destroy_process_group()


def test_sharded_collectives_gloo_ws2():
    ws = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, ws, port, q)) for r in range(ws)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(120)
    res = dict(q.get(timeout=10) for _ in range(ws))
    assert res == {0: "ok", 1: "ok"}, res


def test_single_process_defaults():
    assert parallel.exclusive_carry(123) == 0
    t = torch.tensor([7])
    assert int(parallel.allreduce_sum_(t).item()) == 7
    assert parallel.shard_range(10, 3) == (30, 10)
