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


class SymmetricKeys:
    """Global selection fused into the evaluation launches (§8e, NVSwitch-native variant): a
    symmetric-memory vector of packed keys (torch.distributed._symmetric_memory); every rank's
    aceso_eval_global applies an atomic MIN of its batch key to rank 0's slot through the
    NVLink peer mapping, so a step needs no collective call. Slots are reset to INT64_MAX
    (`reset`, then a barrier) before the steps that use them; `read` after every rank's
    launches have completed (stream synchronised + barrier)."""

    def __init__(self, n_slots: int, group=None):
        import torch.distributed._symmetric_memory as symm
        self.group = group or dist.group.WORLD
        self.buf = symm.empty(int(n_slots), dtype=torch.int64, device=torch.device("cuda", torch.cuda.current_device()))
        self.handle = symm.rendezvous(self.buf, self.group)
        self.root = int(self.handle.buffer_ptrs[0])  # rank 0's buffer, mapped into this rank
        self.rank = dist.get_rank(self.group)

    def slot(self, s: int) -> int:
        """Device address of slot s on rank 0 (valid in this rank's kernels)."""
        return self.root + 8 * int(s)

    def reset(self):
        if self.rank == 0:
            self.buf.fill_((1 << 63) - 1)
        torch.cuda.synchronize()
        dist.barrier(group=self.group)

    def read(self, s: int) -> int:
        """Rank 0: the job-wide packed key of slot s."""
        return int(self.buf[s].item())
