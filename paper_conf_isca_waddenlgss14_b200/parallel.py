"""Multi-GPU data sharding, one process per GPU.

The kernels partition by data: rank r of G owns the contiguous slice
[r*n, (r+1)*n) of the global index space (weak scaling: n fixed per GPU).
Inputs are a pure function of (seed, global index) (inputs.py), so shards need
no transfer.  RMT replicas never span GPUs: the sphere of replication is
on-chip.  The only data-path collectives are the ones the method needs:

  * all-reduce(SUM) of the u64 error counters,
  * all-reduce(SUM) of the Reduction result,
  * all-gather of the PrefixSum shard totals -> each rank's carry-in (the
    exclusive prefix of the earlier shards), passed to the scan kernel.

torch.distributed is plumbing only (NCCL on GPUs; gloo in the CPU tests).
"""
from __future__ import annotations

import torch
import torch.distributed as dist

U32 = 1 << 32


def world() -> tuple[int, int]:
    if dist.is_available() and dist.is_initialized():
        return dist.get_world_size(), dist.get_rank()
    return 1, 0


def shard_range(n_per_rank: int, rank: int) -> tuple[int, int]:
    """(global offset, count) of rank's shard under weak scaling."""
    return rank * n_per_rank, n_per_rank


def allreduce_sum_(t: torch.Tensor, group=None) -> torch.Tensor:
    """In-place SUM all-reduce (error counters, the Reduction result)."""
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
    return t


def exclusive_carry(local_total: int, group=None, device=None) -> int:
    """u32 carry-in of this rank's scan: (sum of the totals of lower ranks) mod 2^32."""
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size(group) == 1:
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


def global_prefixsum(x_local, y_local, s_tmp, err, rmt_mod, variant="none", ws_red=None, ws_ps=None, group=None):
    """Inclusive scan of the concatenation of all ranks' x (mod 2^32): local
    total (Reduction kernel) -> all-gather -> carry-in -> scan kernel."""
    n = x_local.numel()
    rmt_mod.launch("reduction", variant, [x_local, s_tmp], n, err, workspace=ws_red)
    total = int(s_tmp.view(torch.int64)[0].item())
    carry = exclusive_carry(total, group, device=x_local.device)
    rmt_mod.launch("prefixsum", variant, [x_local, y_local], n, err, dims=(carry,), workspace=ws_ps)
    return carry
