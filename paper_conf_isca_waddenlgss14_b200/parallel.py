"""Multi-GPU data sharding, one process per GPU.

The kernels partition by data: rank r of G owns a contiguous slice of the
global index space (weak scaling: the per-rank size is fixed; strong scaling
for BASELINE.json configs[4]: a fixed global size split G ways).  Inputs are a
pure function of (seed, global index) (inputs.py), so shards need no transfer.
RMT replicas never span GPUs: the sphere of replication is on-chip.
The only data-path collectives are the exchanges the kernels themselves need
(SURVEY.md:598-612):

  * all-reduce(SUM) of the u64 error counters (once per measured batch);
  * Reduction: all-reduce(SUM) of the u64 shard sums;
  * PrefixSum: all-gather of the shard totals (u64, on the device); the scan
    kernel adds the lower ranks' totals to its carry on the device;
  * FWT: local FWHT of N/G, then log2 G cross-shard butterfly stages: stage h
    pairs rank r with r ^ (h / (N/G)); the pair swaps shards (send/recv) and
    each runs the RMT-protected combine kernel (x + p below, p - x above: the
    single-GPU stage's own fp32 operations, so the result is bitwise the
    single-GPU one);
  * Sobel: row blocks with a one-row halo above and below (generated locally
    from the index RNG), so shard edges see their true neighbours;
  * Transpose / DCT / BlackScholes / BinarySearch (queries) / MatMul (rows of A
    and C, B replicated): independent, error counters only.
  FloydWarshall does not shard (replicas only: a row-block version needs a
  per-k broadcast of row k, 4096 tiny latency-bound broadcasts).

torch.distributed is plumbing only: NCCL on GPUs (device tensors), gloo in the
CPU tests and in the two-ranks-on-one-GPU test (tensors staged through the
host; that path exists for testing only).
"""
from __future__ import annotations

import torch
import torch.distributed as dist

U32 = 1 << 32


def world() -> tuple[int, int]:
    if dist.is_available() and dist.is_initialized():
        return dist.get_world_size(), dist.get_rank()
    return 1, 0


def _active(group=None) -> bool:
    return dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1


def _host_staged(group=None) -> bool:
    """gloo cannot reduce device tensors: stage through the host."""
    return dist.get_backend(group) == "gloo"


def shard_range(n_per_rank: int, rank: int) -> tuple[int, int]:
    """(global offset, count) of rank's shard under weak scaling."""
    return rank * n_per_rank, n_per_rank


def strong_range(n_total: int, world_size: int, rank: int, align: int = 1) -> tuple[int, int]:
    """(global offset, count) of rank's shard when a fixed global size is split
    world_size ways (strong scaling); shard boundaries are multiples of `align`."""
    units = n_total // align
    lo = units * rank // world_size
    hi = units * (rank + 1) // world_size
    return lo * align, (hi - lo) * align


def allreduce_sum_(t: torch.Tensor, group=None) -> torch.Tensor:
    """In-place SUM all-reduce (error counters, the Reduction result)."""
    if _active(group):
        if _host_staged(group):
            h = t.cpu()
            dist.all_reduce(h, op=dist.ReduceOp.SUM, group=group)
            t.copy_(h)
        else:
            dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
    return t


def all_gather_(out: torch.Tensor, local: torch.Tensor, group=None) -> torch.Tensor:
    """out[r * local.numel() : ...] <- rank r's `local` (device tensors)."""
    if not _active(group):
        out.copy_(local.reshape(-1))
        return out
    if _host_staged(group):
        lst = [torch.empty_like(local, device="cpu") for _ in range(dist.get_world_size(group))]
        dist.all_gather(lst, local.cpu(), group=group)
        out.copy_(torch.cat([t.reshape(-1) for t in lst]))
    else:
        dist.all_gather_into_tensor(out, local, group=group)
    return out


def sendrecv_(send: torch.Tensor, recv: torch.Tensor, peer: int, group=None) -> torch.Tensor:
    """Swap a buffer with rank `peer` (recv <- peer's send)."""
    if _host_staged(group):
        hs, hr = send.cpu(), torch.empty_like(recv, device="cpu")
        ops = [dist.P2POp(dist.isend, hs, peer, group), dist.P2POp(dist.irecv, hr, peer, group)]
        for r in dist.batch_isend_irecv(ops):
            r.wait()
        recv.copy_(hr)
        return recv
    ops = [dist.P2POp(dist.isend, send, peer, group), dist.P2POp(dist.irecv, recv, peer, group)]
    for r in dist.batch_isend_irecv(ops):
        r.wait()
    return recv


def exclusive_carry(local_total: int, group=None, device=None) -> int:
    """u32 carry-in of this rank's scan from a host value (host-side helper;
    the timed path uses global_prefixsum's device all-gather instead)."""
    if not _active(group):
        return 0
    ws = dist.get_world_size(group)
    rk = dist.get_rank(group)
    mine = torch.tensor([int(local_total) % U32], dtype=torch.int64, device=device)
    allv = [torch.zeros_like(mine) for _ in range(ws)]
    dist.all_gather(allv, mine, group=group)
    return int(sum(int(v.item()) for v in allv[:rk])) % U32


def global_reduction(x_local, s_out, err, rmt_mod, variant="none", workspace=None, group=None):
    """s_out[0] <- sum over all ranks' x (exact u64): local Reduction kernel,
    then all-reduce(SUM) of the 8-byte result."""
    rmt_mod.launch("reduction", variant, [x_local, s_out], x_local.numel(), err, workspace=workspace)
    return allreduce_sum_(s_out.view(torch.int64), group)


def global_prefixsum(x_local, y_local, s_tmp, totals, err, rmt_mod, variant="none", ws_red=None, ws_ps=None,
                     group=None):
    """Inclusive scan of the concatenation of all ranks' x (mod 2^32): local
    total (Reduction kernel, u64 on the device) -> all-gather of the G totals
    (device tensor `totals`, int64[G]) -> the scan kernel adds totals[0..rank)
    to its carry on the device.  No host round trip on the NCCL path."""
    n = x_local.numel()
    ws, rk = world() if group is None else (dist.get_world_size(group), dist.get_rank(group))
    rmt_mod.launch("reduction", variant, [x_local, s_tmp], n, err, workspace=ws_red)
    all_gather_(totals, s_tmp.view(torch.int64)[:1], group)
    return rmt_mod.launch("prefixsum", variant, [x_local, y_local, totals], n, err, dims=(0, rk), workspace=ws_ps)


def fwt_partner_stages(world_size: int):
    """Cross-shard stages of a G-way FWT: the partner offset of each stage, in
    the single-GPU stage order (h = N/G, 2N/G, ..., N/2)."""
    out, s = [], 1
    while s < world_size:
        out.append(s)
        s <<= 1
    return out


def global_fwt(x_local, y_local, recv, tmp, err, rmt_mod, variant="none", workspace=None, ws_comb=None, group=None):
    """y_local <- this rank's slice of the FWT of the concatenation of every
    rank's x (G a power of two): local transform, then log2 G cross-shard
    butterfly stages (send/recv with the partner + the RMT combine kernel)."""
    n = x_local.numel()
    ws, rk = world() if group is None else (dist.get_world_size(group), dist.get_rank(group))
    if ws & (ws - 1):
        raise ValueError("global FWT needs a power-of-two number of ranks")
    k = rmt_mod.launch("fwt", variant, [x_local, y_local], n, err, dims=(0,), workspace=workspace)
    for s in fwt_partner_stages(ws):
        peer = rk ^ s
        sendrecv_(y_local, recv, peer, group)
        k += rmt_mod.launch("fwt", variant, [y_local, tmp, recv], n, err, dims=(1, 1 if rk > peer else 0),
                            workspace=ws_comb)
        y_local.copy_(tmp)
    return k


def device_barrier(group=None, device=None):
    """Every rank's previously launched kernels complete before any rank's next
    ones start: a one-element NCCL all-reduce is stream-ordered on every rank (no
    host wait); gloo (tests) synchronises the device and meets on the host."""
    if not _active(group):
        return
    if _host_staged(group):
        torch.cuda.synchronize()
        dist.barrier(group=group)
    else:
        t = torch.zeros(1, dtype=torch.int32, device=device or "cuda")
        dist.all_reduce(t, group=group)


class PeerFWT:
    """The fused multi-GPU FWT: each rank
    keeps two shard buffers and exports both as CUDA IPC handles once; every
    cross-shard stage runs the RMT combine kernel with the PARTNER's current
    buffer as its input p -- peer-to-peer loads over NVLink, so the exchange
    and the butterfly are one kernel and no staged copy is made.  Stage s reads
    buffer cur of both ranks and writes buffer 1 - cur; a device barrier before
    each stage makes the partner's writes of cur visible, and one after the last
    stage keeps a rank from reusing a buffer its partner may still be reading."""

    def __init__(self, n: int, rmt_mod, group=None, device="cuda"):
        self.n, self.rmt, self.group = n, rmt_mod, group
        self.ws, self.rk = world() if group is None else (dist.get_world_size(group), dist.get_rank(group))
        if self.ws & (self.ws - 1):
            raise ValueError("global FWT needs a power-of-two number of ranks")
        self.buf = [torch.empty(n, dtype=torch.float32, device=device) for _ in range(2)]
        mine = [rmt_mod.ipc_export(b) for b in self.buf]
        allh = [None] * self.ws
        if _active(group):
            dist.all_gather_object(allh, mine, group=group)
        else:
            allh = [mine]
        self.peer, self._opened = {}, {}
        for s in fwt_partner_stages(self.ws):
            q = self.rk ^ s
            views = []
            for h, off in allh[q]:
                # both buffers may live in one allocation: a handle is opened once
                if h not in self._opened:
                    self._opened[h] = rmt_mod.ipc_open(h, 0, 0)
                views.append(rmt_mod.DevPtr(self._opened[h].ptr + off, 4 * n))
            self.peer[q] = views

    def close(self):
        for d in self._opened.values():
            self.rmt.ipc_close(d)
        self.peer, self._opened = {}, {}

    def run(self, x_local, err, variant="none", workspace=None, ws_comb=None):
        """Returns (this rank's slice of the global transform, kernels launched)."""
        k = self.rmt.launch("fwt", variant, [x_local, self.buf[0]], self.n, err, dims=(0,), workspace=workspace)
        cur = 0
        for s in fwt_partner_stages(self.ws):
            q = self.rk ^ s
            device_barrier(self.group)
            k += self.rmt.launch("fwt", variant, [self.buf[cur], self.buf[1 - cur], self.peer[q][cur]], self.n, err,
                                 dims=(1, 1 if self.rk > q else 0), workspace=ws_comb)
            cur = 1 - cur
        device_barrier(self.group)
        return self.buf[cur], k


def sobel_halo_rows(H_total: int, r0: int, r1: int) -> tuple[int, int]:
    """Input rows [lo, hi) a rank owning output rows [r0, r1) of an H_total-row
    image needs: one halo row above and below, clipped at the image border (the
    image border rows stay the kernel's own border rows, written 0)."""
    return max(0, r0 - 1), min(H_total, r1 + 1)
