"""Reference copy of the search driver's primitive generator as first written (one
numpy pass per candidate). tests/test_search_cpu.py checks that the optimised generator in
paper_conf_eurosys_liumlsmybw24_b200/search.py produces exactly the same candidates."""
import math

import numpy as np

INFO_OOM = 1 << 16


def stages_of(codes):
    heads = np.flatnonzero(codes & 1)
    ends = np.append(heads[1:], len(codes))
    return heads, ends


def _move_front(codes, s, k):
    """dec-op# of stage s / inc-op# of s-1: first k ops of stage s join stage s-1."""
    heads, ends = stages_of(codes)
    a, e = heads[s], ends[s]
    if s == 0 or k < 1 or k >= e - a:
        return None
    c = codes.copy()
    prev = c[a - 1] & 0xEE
    c[a:a + k] = (c[a:a + k] & 0x10) | prev
    c[a + k] = (c[a + k] & 0xFE) | 1
    return c


def _move_back(codes, s, k):
    """dec-op# of stage s / inc-op# of s+1: last k ops of stage s join stage s+1."""
    heads, ends = stages_of(codes)
    p = len(heads)
    a, e = heads[s], ends[s]
    if s >= p - 1 or k < 1 or k >= e - a:
        return None
    c = codes.copy()
    nxt = c[e] & 0xEE
    c[e] &= 0xFE
    c[e - k:e] = (c[e - k:e] & 0x10) | nxt
    c[e - k] |= 1
    return c


def _recode_stage(codes, s, dt, dd, from_op=None):
    heads, ends = stages_of(codes)
    a, e = heads[s], ends[s]
    lo = a if from_op is None else from_op
    c = codes.copy()
    tpl = ((c[lo:e] >> 1) & 7).astype(np.int16) + dt
    dpl = ((c[lo:e] >> 5) & 7).astype(np.int16) + dd
    if tpl.min() < 0 or dpl.min() < 0 or tpl.max() > 7 or dpl.max() > 7:
        return None
    c[lo:e] = (c[lo:e] & 0x11) | ((tpl.astype(np.uint8) & 7) << 1) | ((dpl.astype(np.uint8) & 7) << 5)
    return c


def _rc_order(prof, codes, s, mbs):
    """Ops of stage s by activation size at their partition, largest first."""
    heads, ends = stages_of(codes)
    a, e = heads[s], ends[s]
    j = np.arange(a, e)
    tpl = (codes[a:e] >> 1) & 7
    dpl = (codes[a:e] >> 5) & 7
    b = np.clip(mbs - dpl.astype(np.int64), 0, prof.n_b - 1)
    act = prof.rec[prof.op_type[a:e], np.minimum(tpl, prof.n_tp - 1), b, 4]
    return j[np.argsort(-act, kind="stable")]


class PrimitivesReference:
    def __init__(self, prof, heuristic2=True, max_k=None):
        self.prof = prof
        self.heuristic2 = heuristic2
        self.max_k = max_k

    def apply_all(self, codes, mbs, info, comp, comm, stage_time):
        """All eligible primitives on the Heuristic-1 bottleneck stage of (codes, mbs).
        Returns a list of (codes, mbs)."""
        prof = self.prof
        heads, ends = stages_of(codes)
        p = len(heads)
        bn = int(info & 0xFF)
        if bn >= p:
            bn = 0
        oom = bool(info & INFO_OOM)
        # Heuristic-2: the resource with the highest consumption proportion of stage bn
        if oom:
            want = {"mem"}
        else:
            cs, ms = max(int(comp[:p].sum()), 1), max(int(comm[:p].sum()), 1)
            want = {"comp"} if comp[bn] / cs >= comm[bn] / ms else {"comm"}
        if not self.heuristic2:
            want = {"mem", "comp", "comm"}
        out = []
        size = ends[bn] - heads[bn]
        kmax = size - 1 if self.max_k is None else min(size - 1, self.max_k)
        # inc/dec-op#: move ops out of the bottleneck at either edge (every resource),
        # with a relay toward the idlest stage
        idle = int(np.argmin(stage_time[:p])) if p > 1 else bn
        for k in range(1, kmax + 1):
            c = _move_front(codes, bn, k)
            if c is not None:
                out.append((c, mbs))
                if idle < bn - 1:
                    c2 = _move_front(c, bn - 1, k)
                    if c2 is not None:
                        out.append((c2, mbs))
            c = _move_back(codes, bn, k)
            if c is not None:
                out.append((c, mbs))
                if idle > bn + 1:
                    c2 = _move_back(c, bn + 1, k)
                    if c2 is not None:
                        out.append((c2, mbs))
        log2bg = int(math.log2(prof.global_batch & -prof.global_batch))
        dmax = int(((codes >> 5) & 7).max())
        # inc/dec-mbs (model level): memory down / computation efficiency up
        if ("mem" in want or "comm" in want) and mbs - 1 >= dmax:
            out.append((codes, mbs - 1))
        if ("comp" in want) and mbs + 1 <= log2bg:
            out.append((codes, mbs + 1))
        # tp <-> dp inside the stage (same devices): inc-tp/dec-dp and dec-tp/inc-dp
        for dt in (1, -1):
            c = _recode_stage(codes, bn, dt, -dt)
            if c is not None:
                out.append((c, max(mbs, int(((c >> 5) & 7).max()))))
        # inc-dp / inc-tp with a partner stage holding twice the devices
        kb = ((codes[heads[bn]] >> 1) & 7) + ((codes[heads[bn]] >> 5) & 7)
        for q in range(p):
            if q == bn:
                continue
            kq = ((codes[heads[q]] >> 1) & 7) + ((codes[heads[q]] >> 5) & 7)
            if kq == kb + 1 and ("comp" in want or "mem" in want):
                for dtb, ddb in ((1, 0), (0, 1)):
                    for dtq, ddq in ((-1, 0), (0, -1)):
                        c = _recode_stage(codes, bn, dtb, ddb)
                        c = _recode_stage(c, q, dtq, ddq) if c is not None else None
                        if c is not None:
                            out.append((c, max(mbs, int(((c >> 5) & 7).max()))))
            if kq + 1 == kb and "comm" in want:  # give devices away (dec-dp/tp on the bottleneck)
                for dtb, ddb in ((-1, 0), (0, -1)):
                    for dtq, ddq in ((1, 0), (0, 1)):
                        c = _recode_stage(codes, bn, dtb, ddb)
                        c = _recode_stage(c, q, dtq, ddq) if c is not None else None
                        if c is not None:
                            out.append((c, max(mbs, int(((c >> 5) & 7).max()))))
        # greedy inc-rc (memory) / dec-rc (computation) on the largest-activation ops
        order = _rc_order(prof, codes, bn, mbs)
        rc = (codes[order] >> 4) & 1
        if "mem" in want:
            todo = order[rc == 0]
            for k in range(1, len(todo) + 1):
                c = codes.copy()
                c[todo[:k]] |= 0x10
                out.append((c, mbs))
        if "comp" in want:
            have = order[rc == 1][::-1]
            for k in range(1, len(have) + 1):
                c = codes.copy()
                c[have[:k]] &= 0xEF
                out.append((c, mbs))
        # op-level fine-tune: tp/dp change from op k to the end of the stage
        for j in range(heads[bn] + 1, ends[bn]):
            for dt in (1, -1):
                c = _recode_stage(codes, bn, dt, -dt, from_op=j)
                if c is not None:
                    out.append((c, max(mbs, int(((c >> 5) & 7).max()))))
        return out


