"""Multi-GPU selection (§8e): shard the candidate batch over ranks, evaluate and
select locally (fused K2 in aceso_eval), then one all-reduce MIN of the packed
64-bit key over NCCL (NVLink / NVSwitch) picks the global winner.

The packed key orders (class, cost, global index) exactly unless the cost field
saturates; a saturated winner triggers an exact fallback (all-gather of every
rank's exact (class<<62 | cost, index) pair, 16 bytes per rank).
"""
from __future__ import annotations

import torch
import torch.distributed as dist

from .api import Selection, decode_key


def shard(n_total: int, rank: int, world: int):
    """Contiguous shard [lo, hi) of rank r: floor(r*n/R) .. floor((r+1)*n/R)."""
    lo = n_total * rank // world
    hi = n_total * (rank + 1) // world
    return lo, hi - lo


def global_select(sel: torch.Tensor, n_total: int, group=None) -> Selection:
    """sel: this rank's select buffer (first 32 bytes = aceso_select_result).

    One all_reduce(MIN) of the int64 key; exact fallback on saturation."""
    key = sel[0:8].view(torch.int64).clone()
    dist.all_reduce(key, op=dist.ReduceOp.MIN, group=group)
    k = int(key.item())
    cls, cost, idx, saturated = decode_key(k, n_total)
    if idx < 0:
        return Selection(-1, 0, -1, k)
    if not saturated:
        return Selection(cls, cost, idx, k)
    pair = sel[8:24].view(torch.int64).clone()
    world = dist.get_world_size(group)
    parts = [torch.empty_like(pair) for _ in range(world)]
    dist.all_gather(parts, pair, group=group)
    best = None
    for p in parts:
        cc = int(p[0].item()) & ((1 << 64) - 1)
        ix = int(p[1].item())
        if ix < 0:
            continue
        if best is None or (cc, ix) < best:
            best = (cc, ix)
    return Selection(best[0] >> 62, best[0] & ((1 << 62) - 1), best[1], k)
