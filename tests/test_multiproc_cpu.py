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
