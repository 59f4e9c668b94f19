"""Thin host search driver: Aceso's iterative bottleneck alleviation (Alg. 1/2,
P:L521-593) on top of the batched evaluator.

The paper estimates one candidate at a time. Here every hop of the
multi-hop search applies all eligible reconfiguration primitives (Table 1,
P:L163-176) with all their argument values to the current frontier, evaluates
them as ONE batch (the evaluator is `aceso_eval`), and keeps the best ones:
  - Heuristic-1: the bottleneck stage comes from the evaluator's info
    word (largest memory if OOM, else longest time);
  - Heuristic-2: the resource with the highest consumption
    proportion (stage share of the total, from the FULL per-stage outputs)
    selects the eligible primitives; "best performance first" orders the
    frontier of the next hop;
  - primitives: inc/dec-op# at both stage edges with relay along neighbours
    (P:L253), inc/dec-mbs, dp/tp trades inside the stage and with a
    partner stage, greedy inc/dec-rc of the largest-activation ops
    (P:L255), op-level tp/dp fine-tuning from op k to the stage end;
  - Alg. 1: restart from the improved config; on failure within MaxHops (7,
    P:L313) continue from GetBestOf(unexplored) (reading R16: keep the
    better of best and new);
  - parallel search per pipeline-stage count: the searches of all
    stage counts are stepped together and share each evaluation batch.
Configurations are deduplicated by their encoding.

The evaluator is any object with `evaluate(codes[n][L] u8, hdr[n] u64) ->
dict(iter, max_mem, info, stage_comp, stage_comm, stage_mem, stage_T [n][G])`:
`GPUEvaluator` below calls libaceso; tests may pass a CPU evaluator.
"""
from __future__ import annotations

import dataclasses
import math
import time

import numpy as np
import torch

INFO_OOM = 1 << 16
INFO_INVALID = 1 << 17


# ---------------------------------------------------------------------------
# configurations (encoding of include/aceso.h)
# ---------------------------------------------------------------------------
def encode(head, tpl, dpl, rc):
    return (head & 1) | ((tpl & 7) << 1) | ((rc & 1) << 4) | ((dpl & 7) << 5)


def header(mbs, p):
    return (mbs & 0xFF) | ((p & 0xFF) << 8)


def stages_of(codes):
    heads = np.flatnonzero(codes & 1)
    ends = np.append(heads[1:], len(codes))
    return heads, ends


def _split_devices(p, G):
    g = [1] * p
    rem = G - p
    while rem > 0:
        cand = [i for i in range(p) if g[i] <= rem]
        if not cand:
            break
        i = min(cand, key=lambda k: g[k])
        rem -= g[i]
        g[i] *= 2
    return [int(math.log2(x)) for x in g]


def initial_config(prof, p, first="dp"):
    """Even partition, balanced devices, minimum microbatch; a stage's devices
    go to data parallelism first (first="dp") or to tensor parallelism first ("tp"), R28."""
    L, G = prof.n_ops, prof.n_devices
    k = _split_devices(p, G)
    if sum(1 << x for x in k) != G:
        return None
    codes = np.zeros(L, np.uint8)
    starts = [L * i // p for i in range(p)] + [L]
    for i in range(p):
        if first == "tp":
            t = min(k[i], prof.n_tp - 1)
            d = k[i] - t
            if d >= prof.n_dp:
                return None
        else:
            d = min(k[i], prof.n_dp - 1)
            t = k[i] - d
        if t >= prof.n_tp:
            return None
        a, b = starts[i], starts[i + 1]
        codes[a:b] = encode(0, t, d, 0)
        codes[a] |= 1
    dmax = int(max((codes >> 5) & 7))
    return codes, dmax


@dataclasses.dataclass
class Result:
    codes: np.ndarray
    mbs: int
    perf: tuple
    iter_ns: int
    max_mem: int
    info: int


def perf_of(info, it, mem):
    """(class, cost): feasible by iteration time before OOM by memory (R12)."""
    if info & INFO_INVALID:
        return (2, 0)
    if info & INFO_OOM:
        return (1, int(mem))
    return (0, int(it))


# ---------------------------------------------------------------------------
# reconfiguration primitives (Table 1) applied to one configuration
# ---------------------------------------------------------------------------
def _move_front(codes, s, k, st=None):
    """dec-op# of stage s / inc-op# of s-1: first k ops of stage s join stage s-1.
    st = stages_of(codes) when the caller has it."""
    heads, ends = stages_of(codes) if st is None else st
    a, e = heads[s], ends[s]
    if s == 0 or k < 1 or k >= e - a:
        return None
    c = codes.copy()
    prev = c[a - 1] & 0xEE
    c[a:a + k] = (c[a:a + k] & 0x10) | prev
    c[a + k] = (c[a + k] & 0xFE) | 1
    return c


def _move_back(codes, s, k, st=None):
    """dec-op# of stage s / inc-op# of s+1: last k ops of stage s join stage s+1."""
    heads, ends = stages_of(codes) if st is None else st
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


def _recode_stage(codes, s, dt, dd, from_op=None, st=None):
    heads, ends = stages_of(codes) if st is None else st
    a, e = heads[s], ends[s]
    lo = a if from_op is None else from_op
    c = codes.copy()
    tpl = ((c[lo:e] >> 1) & 7).astype(np.int16) + dt
    dpl = ((c[lo:e] >> 5) & 7).astype(np.int16) + dd
    if tpl.min() < 0 or dpl.min() < 0 or tpl.max() > 7 or dpl.max() > 7:
        return None
    c[lo:e] = (c[lo:e] & 0x11) | ((tpl.astype(np.uint8) & 7) << 1) | ((dpl.astype(np.uint8) & 7) << 5)
    return c


def _rc_order(prof, codes, s, mbs, st=None):
    """Ops of stage s by activation size at their partition, largest first."""
    heads, ends = stages_of(codes) if st is None else st
    a, e = heads[s], ends[s]
    j = np.arange(a, e)
    tpl = (codes[a:e] >> 1) & 7
    dpl = (codes[a:e] >> 5) & 7
    b = np.clip(mbs - dpl.astype(np.int64), 0, prof.n_b - 1)
    act = prof.rec[prof.op_type[a:e], np.minimum(tpl, prof.n_tp - 1), b, 4]
    return j[np.argsort(-act, kind="stable")]


RESOURCES = ("comp", "comm", "mem")


def resource_order(info, comp, comm, mem, p, bn):
    """Heuristic-2: the bottleneck stage's resources by consumption proportion
    (its consumption divided by the consumption of all stages), highest first; an OOM
    configuration puts memory first (Heuristic-1's safety-first priority). Without
    per-stage memory (mem None) only computation and communication are ranked."""
    shares = {"comp": int(comp[bn]) / max(int(comp[:p].sum()), 1),
              "comm": int(comm[bn]) / max(int(comm[:p].sum()), 1)}
    if mem is not None:
        shares["mem"] = int(mem[bn]) / max(int(mem[:p].sum()), 1)
    order = sorted(shares, key=lambda r: -shares[r])  # stable: comp, comm, mem on ties
    if info & INFO_OOM:
        order = ["mem"] + [r for r in order if r != "mem"]
    return order


def bottleneck_rank(info, mem, stage_time, p, rank):
    """The stage of Heuristic-1's order at `rank` (0: the bottleneck of the info word; 1: the
    secondary bottleneck): stages by memory if OOM, else by time, highest first,
    lowest index on ties."""
    if rank == 0 or p <= 1:
        return int(info & 0xFF)
    key = mem if info & INFO_OOM else stage_time
    order = sorted(range(p), key=lambda i: (-int(key[i]), i))
    return order[min(rank, p - 1)]


class Primitives:
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
        st = (heads, ends)
        for k in range(1, kmax + 1):
            c = _move_front(codes, bn, k, st)
            if c is not None:
                out.append((c, mbs))
                if idle < bn - 1:
                    # stage bn-1 of c: heads unchanged below bn, its end moved by k
                    h2, e2 = heads.copy(), ends.copy()
                    h2[bn] += k
                    e2[bn - 1] += k
                    c2 = _move_front(c, bn - 1, k, (h2, e2))
                    if c2 is not None:
                        out.append((c2, mbs))
            c = _move_back(codes, bn, k, st)
            if c is not None:
                out.append((c, mbs))
                if idle > bn + 1:
                    h2, e2 = heads.copy(), ends.copy()
                    h2[bn + 1] -= k
                    e2[bn] -= k
                    c2 = _move_back(c, bn + 1, k, (h2, e2))
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
            c = _recode_stage(codes, bn, dt, -dt, st=st)
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
                        c = _recode_stage(codes, bn, dtb, ddb, st=st)
                        c = _recode_stage(c, q, dtq, ddq, st=st) if c is not None else None
                        if c is not None:
                            out.append((c, max(mbs, int(((c >> 5) & 7).max()))))
            if kq + 1 == kb and "comm" in want:  # give devices away (dec-dp/tp on the bottleneck)
                for dtb, ddb in ((-1, 0), (0, -1)):
                    for dtq, ddq in ((1, 0), (0, 1)):
                        c = _recode_stage(codes, bn, dtb, ddb, st=st)
                        c = _recode_stage(c, q, dtq, ddq, st=st) if c is not None else None
                        if c is not None:
                            out.append((c, max(mbs, int(((c >> 5) & 7).max()))))
        # greedy inc-rc (memory) / dec-rc (computation) on the largest-activation ops
        order = _rc_order(prof, codes, bn, mbs, st)
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
        a, e = int(heads[bn]), int(ends[bn])
        if e - a > 1:
            # suffix extrema of the stage's tp/dp fields decide which shifts stay in range
            tp = ((codes[a:e] >> 1) & 7).astype(np.int16)
            dp = ((codes[a:e] >> 5) & 7).astype(np.int16)
            tmin, tmax = np.minimum.accumulate(tp[::-1])[::-1], np.maximum.accumulate(tp[::-1])[::-1]
            dmin, dmax_s = np.minimum.accumulate(dp[::-1])[::-1], np.maximum.accumulate(dp[::-1])[::-1]
            dmax_pre = int(((codes[:a] >> 5) & 7).max()) if a > 0 else 0
            dmax_post = int(((codes[e:] >> 5) & 7).max()) if e < len(codes) else 0
            dmax_out = max(dmax_pre, dmax_post)
            for j in range(a + 1, e):
                r = j - a
                for dt in (1, -1):
                    if tmin[r] + dt < 0 or tmax[r] + dt > 7 or dmin[r] - dt < 0 or dmax_s[r] - dt > 7:
                        continue
                    c = codes.copy()
                    seg = c[j:e]
                    c[j:e] = (seg & 0x11) | (((tp[r:] + dt).astype(np.uint8) & 7) << 1) | \
                        (((dp[r:] - dt).astype(np.uint8) & 7) << 5)
                    dnew = max(dmax_out, int(((codes[a:j] >> 5) & 7).max()), int(dmax_s[r] - dt))
                    out.append((c, max(mbs, dnew)))
        return out


    def describe_all(self, codes, mbs, info, comp, comm, stage_time, mem=None, bn=None, resource=None):
        """The candidates of apply_all, in the same order, as base + patches
        (candidates.CAND_DTYPE rows with base = 0) plus the two rank rows of this base
        used by the recompute patches. Nothing is materialised on the host; the families
        with one candidate per op (op moves, recompute ranks, fine-tune starts) are built as
        arrays (numpy), the few others one by one."""
        from . import candidates as C
        prof = self.prof
        L = len(codes)
        heads, ends = stages_of(codes)
        p = len(heads)
        if bn is None:
            bn = int(info & 0xFF)
        if bn >= p:
            bn = 0
        oom = bool(info & INFO_OOM)
        if resource is not None:
            want = {resource}
        elif mem is not None:
            want = {resource_order(info, comp, comm, mem, p, bn)[0]}
        elif oom:
            want = {"mem"}
        else:
            cs, ms = max(int(comp[:p].sum()), 1), max(int(comm[:p].sum()), 1)
            want = {"comp"} if comp[bn] / cs >= comm[bn] / ms else {"comm"}
        if not self.heuristic2:
            want = {"mem", "comp", "comm"}
        groups = []  # (mbs [n], patches [n][MAX_PATCH] PATCH_DTYPE, n_patch [n]) in emission order

        def block(mbs_v, pts):
            """n candidates sharing a patch structure: pts = list of per-slot patch columns,
            each a tuple of arrays/scalars (a, b, kind, v0, v1, v2) broadcast to n."""
            n = len(mbs_v)
            pa = np.zeros((n, C.MAX_PATCH), C.PATCH_DTYPE)
            for j, (pa_, pb_, kind, v0, v1, v2) in enumerate(pts):
                pa["a"][:, j], pa["b"][:, j], pa["kind"][:, j] = pa_, pb_, kind
                pa["v0"][:, j], pa["v1"][:, j], pa["v2"][:, j] = v0, v1, v2
            groups.append((np.asarray(mbs_v, np.uint8), pa, np.full(n, len(pts), np.uint8)))

        def one(m, patches):
            block([m], [tuple(np.array([x]) for x in pt) for pt in patches])

        a, e = int(heads[bn]), int(ends[bn])
        size = e - a
        kmax = size - 1 if self.max_k is None else min(size - 1, self.max_k)
        idle = int(np.argmin(stage_time[:p])) if p > 1 else bn
        if kmax >= 1:
            # op moves at both edges of the bottleneck, relayed toward the idlest
            # stage; per k in the order front, front relay, back, back relay
            k = np.arange(1, kmax + 1)
            M, F = C.PATCH_MASK, 0
            fam = []
            if bn > 0:
                pf = [(a, a + k, M, 0x10, int(codes[a - 1]) & 0xEE, F), (a + k, a + k + 1, M, 0xFE, 1, F)]
                fam.append(pf)
                if idle < bn - 1:
                    a2 = int(heads[bn - 1])
                    fam.append(pf + [(a2, a2 + k, M, 0x10, int(codes[a2 - 1]) & 0xEE, F),
                                     (a2 + k, a2 + k + 1, M, 0xFE, 1, F)])
            if bn < p - 1:
                pb = [(e, e + 1, M, 0xFE, 0, F), (e - k, e, M, 0x10, int(codes[e]) & 0xEE, F),
                      (e - k, e - k + 1, M, 0xFF, 1, F)]
                fam.append(pb)
                if idle > bn + 1:
                    e2 = int(ends[bn + 1])
                    fam.append(pb + [(e2, e2 + 1, M, 0xFE, 0, F), (e2 - k, e2, M, 0x10, int(codes[e2]) & 0xEE, F),
                                     (e2 - k, e2 - k + 1, M, 0xFF, 1, F)])
            if fam:
                nf, nk = len(fam), len(k)
                pa = np.zeros((nk, nf, C.MAX_PATCH), C.PATCH_DTYPE)
                npch = np.zeros((nk, nf), np.uint8)
                for fi, pts in enumerate(fam):
                    npch[:, fi] = len(pts)
                    for j, (pa_, pb_, kind, v0, v1, v2) in enumerate(pts):
                        pa["a"][:, fi, j], pa["b"][:, fi, j], pa["kind"][:, fi, j] = pa_, pb_, kind
                        pa["v0"][:, fi, j], pa["v1"][:, fi, j], pa["v2"][:, fi, j] = v0, v1, v2
                groups.append((np.full(nk * nf, mbs, np.uint8), pa.reshape(nk * nf, C.MAX_PATCH),
                               npch.reshape(-1)))
        log2bg = int(math.log2(prof.global_batch & -prof.global_batch))
        dpl_all = ((codes >> 5) & 7).astype(np.int16)
        tpl_all = ((codes >> 1) & 7).astype(np.int16)
        dmax = int(dpl_all.max())
        if ("mem" in want or "comm" in want) and mbs - 1 >= dmax:
            one(mbs - 1, [])
        if ("comp" in want) and mbs + 1 <= log2bg:
            one(mbs + 1, [])

        # per-stage extrema of the tp / dp fields (one reduceat each)
        st_tmin = np.minimum.reduceat(tpl_all, heads).tolist()
        st_tmax = np.maximum.reduceat(tpl_all, heads).tolist()
        st_dmin = np.minimum.reduceat(dpl_all, heads).tolist()
        st_dmax = np.maximum.reduceat(dpl_all, heads).tolist()

        def stage_ok(sg, dt, dd):
            return (st_tmin[sg] + dt >= 0 and st_tmax[sg] + dt <= 7 and st_dmin[sg] + dd >= 0
                    and st_dmax[sg] + dd <= 7)

        def dmax_after(changes):  # max dp field after per-stage shifts {stage: dd}
            return max(st_dmax[sg] + changes.get(sg, 0) for sg in range(p))
        for dt in (1, -1):
            if stage_ok(bn, dt, -dt):
                one(max(mbs, dmax_after({bn: -dt})), [C.add(a, e, dt, -dt)])
        kb = ((int(codes[heads[bn]]) >> 1) & 7) + ((int(codes[heads[bn]]) >> 5) & 7)
        for q in range(p):
            if q == bn:
                continue
            kq = ((int(codes[heads[q]]) >> 1) & 7) + ((int(codes[heads[q]]) >> 5) & 7)
            trades = []
            if kq == kb + 1 and ("comp" in want or "mem" in want):
                trades = [(dtb, ddb, dtq, ddq) for dtb, ddb in ((1, 0), (0, 1)) for dtq, ddq in ((-1, 0), (0, -1))]
            if kq + 1 == kb and "comm" in want:
                trades += [(dtb, ddb, dtq, ddq) for dtb, ddb in ((-1, 0), (0, -1)) for dtq, ddq in ((1, 0), (0, 1))]
            for dtb, ddb, dtq, ddq in trades:
                if stage_ok(bn, dtb, ddb) and stage_ok(q, dtq, ddq):
                    qa, qe = int(heads[q]), int(ends[q])
                    one(max(mbs, dmax_after({bn: ddb, q: ddq})), [C.add(a, e, dtb, ddb), C.add(qa, qe, dtq, ddq)])
        stride = C.stride_of(L)
        ranks = np.full((2, stride), 0xFFFF, np.uint16)
        order = _rc_order(prof, codes, bn, mbs, (heads, ends))
        rc = (codes[order] >> 4) & 1
        R = C.PATCH_RANK_RC
        if "mem" in want:
            todo = order[rc == 0]
            ranks[0, todo] = np.arange(len(todo), dtype=np.uint16)
            if len(todo):
                k = np.arange(1, len(todo) + 1)
                block(np.full(len(k), mbs), [(a, e, R, k & 0xFF, (k >> 8) & 0xFF, 0)])
        if "comp" in want:
            have = order[rc == 1][::-1]
            ranks[1, have] = np.arange(len(have), dtype=np.uint16)
            if len(have):
                k = np.arange(1, len(have) + 1)
                block(np.full(len(k), mbs), [(a, e, R, k & 0xFF, (k >> 8) & 0xFF, 1 | 2)])
        if e - a > 1:
            tp, dp = tpl_all[a:e], dpl_all[a:e]
            tmin, tmax = np.minimum.accumulate(tp[::-1])[::-1], np.maximum.accumulate(tp[::-1])[::-1]
            dmin, dmax_s = np.minimum.accumulate(dp[::-1])[::-1], np.maximum.accumulate(dp[::-1])[::-1]
            dmax_pre = int(dpl_all[:a].max()) if a > 0 else 0
            dmax_post = int(dpl_all[e:].max()) if e < L else 0
            dmax_out = max(dmax_pre, dmax_post)
            pmax = np.maximum.accumulate(dp)  # pmax[r - 1] = max dp over [a, a + r)
            r = np.arange(1, e - a)
            js, dts, ms_ = [], [], []
            for dt in (1, -1):  # interleaved per j below: (j, +1), (j, -1)
                ok = ~((tmin[r] + dt < 0) | (tmax[r] + dt > 7) | (dmin[r] - dt < 0) | (dmax_s[r] - dt > 7))
                dnew = np.maximum(np.maximum(dmax_out, pmax[r - 1]), dmax_s[r] - dt)
                js.append(np.where(ok, r, -1))
                dts.append(np.full(len(r), dt))
                ms_.append(np.maximum(mbs, dnew))
            jj = np.stack(js, 1).reshape(-1)
            dd = np.stack(dts, 1).reshape(-1)
            mm = np.stack(ms_, 1).reshape(-1)
            keep = jj >= 0
            jj, dd, mm = jj[keep] + a, dd[keep], mm[keep]
            if len(jj):
                block(mm, [(jj, e, C.PATCH_ADD, dd & 0xFF, (-dd) & 0xFF, 0)])
        if not groups:
            return np.zeros(0, C.CAND_DTYPE), ranks
        n = sum(len(g[0]) for g in groups)
        cands = np.zeros(n, C.CAND_DTYPE)
        cands["mbs"] = np.concatenate([g[0] for g in groups])
        cands["p"] = p
        cands["n_patch"] = np.concatenate([g[2] for g in groups])
        cands["patch"] = np.concatenate([g[1] for g in groups])
        return cands, ranks


# ---------------------------------------------------------------------------
# evaluators
# ---------------------------------------------------------------------------
class GPUEvaluator:
    """aceso_eval in FULL mode on the device; uploads row-major codes and packs them."""

    def __init__(self, ctx):
        self.ctx = ctx
        self.calls = 0
        self.evaluated = 0
        self._tiled = None  # expand output, reused across batches (grown on demand)
        self._flat = None   # FULL outputs of evaluate_cands, reused across batches

    def _outputs(self, n):
        """FULL output arrays for n candidates as views of one reused flat device buffer (the
        search copies what it keeps before the next batch overwrites them)."""
        from .api import Outputs
        pm = self.ctx.n_devices
        need = n * (3 + 4 * pm)  # int64 words: iter, max_mem, info (as int64 slot), 4 stage arrays
        if self._flat is None or self._flat.numel() < need:
            self._flat = torch.empty(max(need, 2 * (0 if self._flat is None else self._flat.numel())),
                                     dtype=torch.int64, device=torch.device("cuda", self.ctx.device))
        f = self._flat
        o = Outputs(f[0:n], f[n:2 * n], f[2 * n:3 * n].view(torch.int32)[0:n])
        o.p_max = pm
        base = 3 * n
        o.stage_T = f[base:base + pm * n].view(pm, n)
        o.stage_mem = f[base + pm * n:base + 2 * pm * n].view(pm, n)
        o.stage_comp = f[base + 2 * pm * n:base + 3 * pm * n].view(pm, n)
        o.stage_comm = f[base + 3 * pm * n:base + 4 * pm * n].view(pm, n)
        return o

    def evaluate(self, codes, hdr, dims=None, hashes=False):
        """Row-major codes [n][L] (+ optional dimension bytes [n][L]) -> FULL outputs
        (+ configuration hashes, aceso_hash)."""
        from .api import as_u32, as_u64, hash_candidates
        n = int(hdr.shape[0])
        self.calls += 1
        self.evaluated += n
        dev = torch.device("cuda", self.ctx.device)
        c = torch.from_numpy(np.ascontiguousarray(codes)).to(dev)
        h = torch.from_numpy(np.ascontiguousarray(hdr, np.uint64).view(np.int64)).to(dev)
        tiled = self.ctx.pack_rowmajor(c)
        plane = None
        if dims is not None:
            plane = self.ctx.pack_dims(torch.from_numpy(np.ascontiguousarray(dims, np.uint8)).to(dev))
        out, _ = self.ctx.eval(tiled, h, n=n, full=True, select=False, dims=plane)
        res = dict(iter=as_u64(out.iter_ns), max_mem=as_u64(out.max_mem), info=as_u32(out.info))
        for k in ["stage_T", "stage_mem", "stage_comp", "stage_comm"]:
            res[k] = as_u64(getattr(out, k)).reshape(out.p_max, n).T
        if hashes:
            hs = hash_candidates(tiled, h, self.ctx.n_ops, n=n)
            res["hash"], res["hash_dev"] = hs.cpu().numpy().view(np.uint64), hs
        return res

    def visited(self):
        """The search's visited set on this device (aceso_dedup)."""
        return DeviceVisited(self.ctx.device)

    def evaluate_cands(self, bases, ranks, cands):
        """Candidates as base + patches: aceso_expand -> aceso_eval (FULL) -> aceso_hash on the
        device; only the descriptors go up (56 B each) and the results come back."""
        from .api import as_u32, as_u64, hash_candidates
        n = int(len(cands))
        self.calls += 1
        self.evaluated += n
        dev = torch.device("cuda", self.ctx.device)
        tb = torch.from_numpy(np.ascontiguousarray(bases)).to(dev)
        rk = torch.from_numpy(np.ascontiguousarray(ranks).view(np.int16)).to(dev)
        cd = torch.from_numpy(np.ascontiguousarray(cands).view(np.uint8)).to(dev)
        from .api import tiled_bytes
        need = int(tiled_bytes(max(n, 1), self.ctx.n_ops))
        if self._tiled is None or self._tiled.numel() < need:
            # aceso_expand writes every byte of the candidates' tiles; lanes past n in the
            # last tile are never read into an output
            self._tiled = torch.empty(max(need, 2 * (0 if self._tiled is None else self._tiled.numel())),
                                      dtype=torch.uint8, device=dev)
        tiled, hdr = self.ctx.expand(tb, cd, rk, n=n, tiled=self._tiled[:need])
        out, _ = self.ctx.eval(tiled, hdr, n=n, full=True, select=False, out=self._outputs(n))
        hs = hash_candidates(tiled, hdr, self.ctx.n_ops, n=n)
        res = dict(iter=as_u64(out.iter_ns), max_mem=as_u64(out.max_mem), info=as_u32(out.info),
                   hash=hs.cpu().numpy().view(np.uint64), hash_dev=hs)
        # per-stage rows stay on the device ([n][p_max] views of the reused buffer, valid until
        # the next call): the search copies the rows of the configurations it may take
        # (Heuristic-2 needs them), not the whole batch
        for k in ["stage_T", "stage_mem", "stage_comp", "stage_comm"]:
            res[k] = getattr(out, k).view(torch.int64).reshape(out.p_max, n).T
        return res


# ---------------------------------------------------------------------------
# Alg. 1 / Alg. 2, batched
# ---------------------------------------------------------------------------
@dataclasses.dataclass
class _Node:
    key: int            # configuration hash (aceso_hash)
    mbs: int
    perf: tuple
    info: int
    comp: np.ndarray
    comm: np.ndarray
    time: np.ndarray
    iter_ns: int
    max_mem: int
    src: tuple | None   # (base row, rank rows, descriptor, n_ops): materialised on demand
    _codes: np.ndarray | None = None
    mem: np.ndarray | None = None  # per-stage memory (Heuristic-2's third resource)

    @property
    def codes(self):
        if self._codes is None:
            from . import candidates as C
            base, ranks, cand, L = self.src
            one = np.array([cand])
            one["base"] = 0  # the single base row passed below
            c, _ = C.expand_host(base[None], ranks[None], one, L)
            self._codes = c[0]
        return self._codes


def _first_new(hs, visited):
    """Configuration dedup: mask of the candidates whose hash is neither in the
    sorted array `visited` nor earlier in `hs` (first occurrence in generation order), and the
    updated sorted array. Sort-based, O(n log n) per batch."""
    keep = np.zeros(len(hs), bool)
    if len(hs) == 0:
        return keep, visited
    order = np.argsort(hs, kind="stable")
    sh = hs[order]
    first = np.empty(len(sh), bool)
    first[0] = True
    first[1:] = sh[1:] != sh[:-1]
    idx, h = order[first], sh[first]
    if len(visited):
        pos = np.searchsorted(visited, h)
        seen = visited[np.minimum(pos, len(visited) - 1)] == h
        idx, h = idx[~seen], h[~seen]
    keep[idx] = True
    return keep, np.insert(visited, np.searchsorted(visited, h), h)


class _HostVisited:
    """Visited set of an evaluator without a device one: sorted host hashes (_first_new)."""

    def __init__(self):
        self.h = np.zeros(0, np.uint64)

    def first_new(self, r):
        keep, self.h = _first_new(np.asarray(r["hash"], np.uint64), self.h)
        return keep


class DeviceVisited:
    """Configuration dedup on the device: every batch's hashes (r["hash_dev"], left
    on the device by aceso_hash) go through aceso_dedup's open-addressing table, first
    occurrence in generation order across batches, the same rule as _first_new. Before the
    load factor would pass 1/2 the table is rebuilt 4x larger from the device list of every
    configuration seen, so the insert never fills it; only the keep mask (1 byte per
    candidate) comes back to the host."""

    def __init__(self, device, slots=1 << 16):
        from .api import VisitedSet
        self._cls = VisitedSet
        self.device = device
        self.vs = VisitedSet(slots, device)
        self.seen = []   # device tensors of first-occurrence hashes (re-inserted on growth)
        self.count = 0

    def _grow(self, need):
        slots = self.vs.slots
        while slots < 4 * need:
            slots *= 2
        self.vs = self._cls(slots, self.device)
        if self.seen:
            self.seen = [torch.cat(self.seen)]
            self.vs.insert(self.seen[0])

    def first_new(self, r):
        hs = r["hash_dev"]
        n = int(hs.shape[0])
        if 2 * (self.count + n) > self.vs.slots:
            self._grow(self.count + n)
        new = self.vs.insert(hs) == 0
        if self.vs.overflowed():
            raise RuntimeError("aceso_dedup: visited table full")  # unreachable at load <= 1/2
        self.seen.append(hs[new])
        keep = new.cpu().numpy()
        self.count += int(keep.sum())
        return keep


def _row(x, i):
    """Row i of a per-stage array, as numpy (device tensors are copied on demand)."""
    return x[i].cpu().numpy().view(np.uint64) if isinstance(x, torch.Tensor) else x[i]


def _key(perf):
    """(class, cost) as one integer with the same order (cost < 2^62)."""
    return (int(perf[0]) << 62) | int(perf[1])


def _keys_of(r):
    info = np.asarray(r["info"], np.uint64)
    cls = np.where(info & INFO_INVALID, 2, np.where(info & INFO_OOM, 1, 0)).astype(np.uint64)
    cost = np.where(cls == 2, 0, np.where(cls == 1, r["max_mem"], r["iter"])).astype(np.uint64)
    return (cls << np.uint64(62)) | cost  # perf_of as one ordered integer


def _oom_excess(r, capacity):
    """Per candidate: sum over its stages of the memory above the capacity, sum_i max(0,
    Mem_i - C), for OOM candidates (0 for the others). The search's tie-break among OOM
    candidates of equal max_i Mem_i (R26): the one closer to feasibility first, so a
    recompute move that fixes the whole bottleneck stage wins over one that only brings it
    down to the next stage's memory."""
    info = np.asarray(r["info"], np.uint64)
    oom = ((info & np.uint64(INFO_OOM)) != 0) & ((info & np.uint64(INFO_INVALID)) == 0)
    ex = np.zeros(len(info), np.int64)
    rows = np.flatnonzero(oom)
    if len(rows) == 0:
        return ex
    sm = r["stage_mem"]
    p = ((info[rows] >> np.uint64(8)) & np.uint64(0xFF)).astype(np.int64)
    if isinstance(sm, torch.Tensor):  # device FULL outputs: reduce there, copy 8 B per row
        dev = sm.device
        rt = torch.from_numpy(rows).to(dev)
        pt = torch.from_numpy(p).to(dev)
        live = torch.arange(sm.shape[1], device=dev)[None, :] < pt[:, None]
        x = torch.clamp(sm[rt] - int(capacity), min=0)
        ex[rows] = torch.where(live, x, torch.zeros_like(x)).sum(dim=1).cpu().numpy()
        return ex
    sm = np.asarray(sm)[rows].view(np.int64)
    live = np.arange(sm.shape[1])[None, :] < p[:, None]
    ex[rows] = np.where(live, np.maximum(sm.astype(np.int64) - int(capacity), 0), 0).sum(axis=1)
    return ex


class _Take:
    """arr[idx[t]] without copying arr (a chunk's view of its batch's arrays)."""
    __slots__ = ("arr", "idx")

    def __init__(self, arr, idx):
        self.arr, self.idx = arr, idx

    def __getitem__(self, t):
        return self.arr[self.idx[t]]

    def rows(self, a, b):
        return self.arr[self.idx[a:b]]


class _Chunk:
    """The configurations one hop added to a search's unexplored set, kept as arrays in
    best-performance-first order (stable: generation order among equals). Nodes are only
    materialised when the search takes them; they leave the set from the front (the
    improving node, the next frontier, GetBestOf)."""

    def __init__(self, keys, idx, r, bases, ranks, cands, L, codes=None, mbs=None, evaluator=None,
                 keep_rows=64):
        self.keys = keys[idx]
        self.idx = idx
        # the batch's arrays, read through idx (entry t = batch row idx[t]); nothing is copied
        self.hash = _Take(r["hash"], idx)
        self.info = _Take(r["info"], idx)
        self.iter = _Take(r["iter"], idx)
        self.mem = _Take(r["max_mem"], idx)
        stage = (r["stage_comp"], r["stage_comm"], r["stage_T"], r["stage_mem"])  # [n][p_max]
        self.cands = None if cands is None else _Take(cands, idx)
        self.codes = None if codes is None else _Take(codes, idx)  # materialised rows (recompute attachment)
        self.mbs = None if mbs is None else _Take(mbs, idx)
        self.bases, self.ranks, self.L = bases, ranks, L
        self.head = 0
        self.evaluator = evaluator
        if isinstance(stage[0], torch.Tensor):
            # device rows (the evaluator's buffer, overwritten by its next batch): copy those of
            # the best `keep_rows` entries, the ones the search takes first; later ones are
            # re-evaluated on demand (node)
            k = min(int(keep_rows), len(idx))
            ti = torch.from_numpy(np.ascontiguousarray(idx[:k])).to(stage[0].device)
            self.rows = torch.stack([x[ti] for x in stage], 1).cpu().numpy().view(np.uint64)  # [k][4][p_max]
            self.stage = None
        else:
            self.rows = None
            self.stage = stage

    def node(self, t):
        info = int(self.info[t])
        i = int(self.idx[t])
        if self.stage is not None:
            rows = [_row(x, i) for x in self.stage]
        elif t < len(self.rows):
            rows = list(self.rows[t])
        else:
            # beyond the copied rows: evaluate this one configuration again (same FULL outputs)
            c1 = self.cands.rows(t, t + 1).copy()
            b1 = int(c1[0]["base"])
            c1["base"] = 0
            r1 = self.evaluator.evaluate_cands(self.bases[b1:b1 + 1], self.ranks[b1:b1 + 1], c1)
            rows = [np.asarray(r1[k][0].cpu().numpy()).view(np.uint64) if isinstance(r1[k], torch.Tensor)
                    else r1[k][0] for k in ("stage_comp", "stage_comm", "stage_T", "stage_mem")]
        if self.codes is not None:
            return _Node(int(self.hash[t]), int(self.mbs[t]), perf_of(info, self.iter[t], self.mem[t]), info,
                         rows[0], rows[1], rows[2], int(self.iter[t]), int(self.mem[t]), None,
                         self.codes[t], rows[3])
        c = self.cands[t]
        b = int(c["base"])
        return _Node(int(self.hash[t]), int(c["mbs"]), perf_of(info, self.iter[t], self.mem[t]), info,
                     rows[0], rows[1], rows[2], int(self.iter[t]), int(self.mem[t]),
                     (self.bases[b], self.ranks[b], c, self.L), None, rows[3])


# the root of a failed multi-hop search is retried on Heuristic-2's next resource (backtracking
# over the primitive groups), then on the secondary bottleneck, before
# GetBestOf(unexplored) (Alg. 1 line 13)
ROOT_MODES = ((0, 0), (0, 1), (0, 2), (1, 0))


class _Search:
    """One AcesoSearch (Alg. 1) for one stage count, stepped one hop at a time."""

    def __init__(self, start: _Node):
        self.cur = start
        self.best = start
        self.init_perf = start.perf
        self.frontier = [start]
        self.hop = 0
        self.mode = 0      # index into ROOT_MODES for the current root
        self.chunks = []   # unexplored configurations, in insertion order (_Chunk)
        self.done = False
        self.improvements = 0
        self.last_best = start.perf  # patience bookkeeping (search())
        self.stale = 0

    def get_best_of_unexplored(self):
        """GetBestOf(unexplored) (Alg. 1): the best remaining configuration, the
        earliest inserted among equals; removed from the set. None if empty."""
        best = None
        for ch in self.chunks:
            if ch.head < len(ch.keys) and (best is None or ch.keys[ch.head] < best.keys[best.head]):
                best = ch
        if best is None:
            return None
        nd = best.node(best.head)
        best.head += 1
        return nd

    def take_best(self, chunks, k):
        """The k best configurations of this hop's chunks (removed from the unexplored set)."""
        out = []
        for _ in range(k):
            best = None
            for ch in chunks:
                if ch.head < len(ch.keys) and (best is None or ch.keys[ch.head] < best.keys[best.head]):
                    best = ch
            if best is None:
                break
            out.append(best.node(best.head))
            best.head += 1
        return out


def _greedy_counts(n):
    """How many ops the greedy recompute steps try: every k up to 16, then k growing by 25%
    (the smallest fitting k of the batch is within 25% of the exact greedy stopping point),
    and all n."""
    ks, k = list(range(1, min(n, 16) + 1)), 16
    while k < n:
        k = min(n, max(k + 1, int(k * 1.25)))
        ks.append(k)
    return ks


def _rc_variants(prof, codes, mbs, info, mem, stage_time, max_n=4096):
    """Recomputation attached to a primitive's result (greedy as in P:L255): on its
    memory bottleneck (if OOM) the largest-activation ops not yet recomputed, the first k in
    order (inc-rc); otherwise on its time bottleneck the recomputed ops released smallest
    activation first (dec-rc); k from _greedy_counts. Returns a list of code rows (same
    header)."""
    heads, ends = stages_of(codes)
    p = len(heads)
    bn = int(info & 0xFF)
    if bn >= p:
        return []
    order = _rc_order(prof, codes, bn, mbs, (heads, ends))
    rc = (codes[order] >> 4) & 1
    out = []
    if info & INFO_OOM:
        todo = order[rc == 0]
        for k in _greedy_counts(min(len(todo), max_n)):
            c = codes.copy()
            c[todo[:k]] |= 0x10
            out.append(c)
    else:
        have = order[rc == 1][::-1]
        for k in _greedy_counts(min(len(have), max_n)):
            c = codes.copy()
            c[have[:k]] &= 0xEF
            out.append(c)
    return out


def search(prof, evaluator, p_values=None, budget_s=10.0, max_hops=7, beam=4, heuristic2=True,
           max_batch=200000, max_k=None, patience=None, starts=None, attach_rc=8, root_modes=ROOT_MODES,
           max_batches=None, init_first=("dp", "tp"), chunk_rows=64):
    """Runs the batched Aceso search. Returns (best Result, stats dict).

    starts: optional extra initial configurations [(codes, mbs_log2)], each searched like the
    paper's initial configurations (e.g. the optimum of the exhaustive stage-uniform space,
    exhaustive.py, for the hybrid of §9b of DESIGN.md).

    Every hop's candidates are generated as base + patches (Primitives.describe_all) and
    evaluated by `evaluator.evaluate_cands(bases, ranks, cands)`, which also returns each
    candidate's configuration hash; configurations are deduplicated by hash in
    generation order (the evaluator's device visited set, `evaluator.visited()`, else the
    host statement), and only the ones the search keeps are materialised on the host.
    attach_rc: per search and hop, the best `attach_rc` new configurations also get greedy
    inc/dec-rc attached (evaluated as rows in a second batch of the hop).
    root_modes: (bottleneck rank, resource rank) tried at the root of a failed multi-hop
    search before GetBestOf: Heuristic-2's next resources, then the secondary bottleneck.
    max_batches: stop after this many evaluation batches (a budget independent of speed).
    patience: a stage count's search stops after this many batches without improving its own
    best (None: only the clock budget, max_batches and exhausted searches stop).
    init_first: the initial configurations per stage count, devices to data parallelism first
    and / or to tensor parallelism first (R28).
    chunk_rows: per hop and search, the per-stage rows of this many best new configurations
    are copied from the device; configurations taken later are evaluated again."""
    from . import candidates as C
    t0 = time.perf_counter()
    L = prof.n_ops
    stride = C.stride_of(L)
    prims = Primitives(prof, heuristic2=heuristic2, max_k=max_k)
    if p_values is None:
        p_values = [p for p in (1, 2, 3, 4, 6, 8, 12, 16, 24, 32, 48, 64) if p <= min(prof.n_devices, prof.n_ops)]
    # every configuration seen: the evaluator's device set, else sorted host hashes
    seen = evaluator.visited() if hasattr(evaluator, "visited") else _HostVisited()
    init = []
    for p in p_values:
        seen_p = []
        for first in init_first:  # R28: both device splits of the paper's initial configuration
            r = initial_config(prof, p, first)
            if r is not None and not any(np.array_equal(r[0], c) for c in seen_p):
                seen_p.append(r[0])
                init.append(r)
    for c, m in (starts or []):
        init.append((np.asarray(c, np.uint8), int(m)))
    bases = np.zeros((len(init), stride), np.uint8)
    ranks = np.full((len(init), 2, stride), 0xFFFF, np.uint16)
    cands = np.zeros(len(init), C.CAND_DTYPE)
    for i, (c, m) in enumerate(init):
        bases[i, :L] = c
        cands[i]["base"], cands[i]["mbs"], cands[i]["p"] = i, m, int((c & 1).sum())
    res = evaluator.evaluate_cands(bases, ranks, cands)
    seen.first_new(res)

    def node(i, r, base_row, rank_rows, cand):
        info = int(r["info"][i])
        nd = _Node(int(r["hash"][i]), int(cand["mbs"]), perf_of(info, r["iter"][i], r["max_mem"][i]), info,
                   _row(r["stage_comp"], i), _row(r["stage_comm"], i), _row(r["stage_T"], i), int(r["iter"][i]),
                   int(r["max_mem"][i]), (base_row, rank_rows, cand, L), None, _row(r["stage_mem"], i))
        return nd

    searches = []
    for i in range(len(init)):
        n0 = node(i, res, bases[i], ranks[i], cands[i])
        n0._codes = init[i][0]
        searches.append(_Search(n0))
    best = min((s.best for s in searches), key=lambda n: n.perf)
    t_best = time.perf_counter() - t0
    batches = 0
    evaluated = len(init)
    history = [(t_best, best.perf)]
    while time.perf_counter() - t0 < budget_s and any(not s.done for s in searches) and \
            (max_batches is None or batches < max_batches):
        # one hop of every active search, generated into one batch of descriptors
        owners, chunks, base_rows, rank_rows = [], [], [], []
        total = 0
        share = max_batch // max(1, sum(1 for s in searches if not s.done))
        for si, s in enumerate(searches):
            if s.done:
                continue
            bn_rank, res_rank = root_modes[s.mode] if s.hop == 0 else (0, 0)
            # every active search (stage count) gets an equal share of the batch, so long
            # models' many-candidate hops cannot starve the later searches
            cap = total + share
            for nd in s.frontier:
                if nd.perf[0] == 2 or total >= cap:
                    continue
                p = int((nd.codes & 1).sum())
                kw = {}
                if nd.mem is not None and heuristic2:
                    bn = bottleneck_rank(nd.info, nd.mem, nd.time, p, bn_rank)
                    order = resource_order(nd.info, nd.comp, nd.comm, nd.mem, p, bn)
                    kw = dict(mem=nd.mem, bn=bn, resource=order[min(res_rank, len(order) - 1)])
                cd, rk = prims.describe_all(nd.codes, nd.mbs, nd.info, nd.comp, nd.comm, nd.time, **kw)
                if len(cd) == 0:
                    continue
                cd = cd[: cap - total]
                cd["base"] = len(base_rows)
                row = np.zeros(stride, np.uint8)
                row[:L] = nd.codes
                base_rows.append(row)
                rank_rows.append(rk)
                chunks.append(cd)
                owners.append(np.full(len(cd), si, np.int32))
                total += len(cd)
        if not chunks:
            for s in searches:
                s.done = True
            break
        bases = np.stack(base_rows)
        ranks = np.stack(rank_rows)
        cands = np.concatenate(chunks)
        r = evaluator.evaluate_cands(bases, ranks, cands)
        batches += 1
        evaluated += len(cands)
        owner = np.concatenate(owners)
        # configurations seen before (or earlier in this batch) are dropped
        keep = seen.first_new(r)
        keys = _keys_of(r)
        ex = _oom_excess(r, prof.mem_capacity)
        hop_chunks = {}
        for si, s in enumerate(searches):
            if s.done:
                continue
            idx = np.nonzero(keep & (owner == si))[0]
            # Heuristic-2: best estimated performance first (stable: generation order)
            idx = idx[np.lexsort((ex[idx], keys[idx]))]  # stable: generation order among equals
            hop_chunks[si] = [_Chunk(keys, idx, r, bases, ranks, cands, L, evaluator=evaluator,
                                      keep_rows=chunk_rows)] if len(idx) else []
        # recomputation attached to the primitives' results: a second batch of the hop
        if attach_rc:
            rows, hdrs, mbss, rowner = [], [], [], []
            for si, chs in hop_chunks.items():
                if not chs:
                    continue
                ch = chs[0]
                for t in range(min(attach_rc, len(ch.keys))):
                    if int(ch.info[t]) & INFO_INVALID:
                        continue
                    nd = ch.node(t)
                    p = int((nd.codes & 1).sum())
                    for c in _rc_variants(prof, nd.codes, nd.mbs, nd.info, nd.mem, nd.time):
                        rows.append(c)
                        hdrs.append(header(nd.mbs, p))
                        mbss.append(nd.mbs)
                        rowner.append(si)
            if rows:
                rc_codes = np.stack(rows)
                rr = evaluator.evaluate(rc_codes, np.array(hdrs, np.uint64), hashes=True)
                batches += 1
                evaluated += len(rows)
                keep2 = seen.first_new(rr)
                keys2 = _keys_of(rr)
                ex2 = _oom_excess(rr, prof.mem_capacity)
                rowner = np.array(rowner)
                mbss = np.array(mbss)
                for si in hop_chunks:
                    idx = np.nonzero(keep2 & (rowner == si))[0]
                    if len(idx):
                        idx = idx[np.lexsort((ex2[idx], keys2[idx]))]
                        hop_chunks[si].append(_Chunk(keys2, idx, rr, None, None, None, L, codes=rc_codes, mbs=mbss))
        for si, s in enumerate(searches):
            if s.done:
                continue
            chs = hop_chunks.get(si, [])
            s.chunks.extend(chs)
            first = min((int(ch.keys[0]) for ch in chs), default=None)
            if first is not None and first < _key(s.init_perf):
                # Alg. 2 returns the improved configuration; Alg. 1 restarts from it
                nd0 = s.take_best(chs, 1)[0]  # leaves the unexplored set
                s.cur = nd0
                if nd0.perf < s.best.perf:
                    s.best = nd0
                s.init_perf = nd0.perf
                s.frontier = [nd0]
                s.hop = 0
                s.mode = 0
                s.improvements += 1
                continue
            s.hop += 1
            if s.hop < max_hops and chs:
                # the next hop explores the best configurations of this one (they leave the
                # unexplored set, Alg. 2 line 1)
                s.frontier = s.take_best(chs, beam)
                continue
            # MultiHop failed within MaxHops: retry the root on the next resource / the
            # secondary bottleneck, then Alg. 1 continues from GetBestOf(unexplored)
            if s.mode + 1 < len(root_modes):
                s.mode += 1
                s.frontier = [s.cur]
                s.hop = 0
                continue
            nd = s.get_best_of_unexplored()
            if nd is None:
                s.done = True
                continue
            s.cur = nd
            s.init_perf = nd.perf
            s.frontier = [nd]
            s.hop = 0
            s.mode = 0
        cur_best = min((s.best for s in searches), key=lambda n: n.perf)
        if cur_best.perf < best.perf:
            best = cur_best
            t_best = time.perf_counter() - t0
            history.append((t_best, best.perf))
        # patience per search (stage count): a search stops after `patience` batches without
        # improving its own best (each stage count is its own Alg. 1 run); the clock
        # budget stops them all
        for s in searches:
            if s.done:
                continue
            if s.best.perf < s.last_best:
                s.last_best = s.best.perf
                s.stale = 0
            else:
                s.stale += 1
                if patience is not None and s.stale >= patience:
                    s.done = True
    total_t = time.perf_counter() - t0
    stats = dict(time_s=total_t, time_to_best_s=t_best, batches=batches, evaluated=evaluated,
                 searches=len(searches), history=history,
                 improvements=sum(s.improvements for s in searches))
    return Result(best.codes, best.mbs, best.perf, best.iter_ns, best.max_mem, best.info), stats


def finetune_dims(prof, evaluator, codes, mbs, dims=None, max_rounds=64):
    """Op-level fine-tuning of the tensor-parallel partition dimension (§4.2):
    "we check the partition options for each operator to determine if there is a better
    dimension". Each round evaluates, as one batch, the configuration with every single op
    whose alternative records differ switched to its other dimension, and keeps the best
    improving switch; stops when none improves. Returns (dims [L] u8, perf, stats)."""
    rec_alt = getattr(prof, "rec_alt", None)
    L = prof.n_ops
    dims = np.zeros(L, np.uint8) if dims is None else np.asarray(dims, np.uint8).copy()
    p = int((codes & 1).sum())
    hdr1 = np.array([header(mbs, p)], np.uint64)
    cur = evaluator.evaluate(codes[None, :], hdr1, dims=dims[None, :])
    perf = perf_of(int(cur["info"][0]), cur["iter"][0], cur["max_mem"][0])
    stats = dict(rounds=0, evaluated=1, switched=[])
    if rec_alt is None:
        return dims, perf, stats
    tpl = np.minimum((codes >> 1) & 7, prof.n_tp - 1)
    b = np.clip(mbs - ((codes >> 5) & 7).astype(np.int64), 0, prof.n_b - 1)
    differs = np.nonzero((rec_alt[prof.op_type, tpl, b] != prof.rec[prof.op_type, tpl, b]).any(axis=1))[0]
    for _ in range(max_rounds):
        if len(differs) == 0:
            break
        cand = np.repeat(dims[None, :], len(differs), axis=0)
        cand[np.arange(len(differs)), differs] ^= 1
        r = evaluator.evaluate(np.repeat(codes[None, :], len(differs), axis=0),
                               np.repeat(hdr1, len(differs)), dims=cand)
        stats["rounds"] += 1
        stats["evaluated"] += len(differs)
        keys = _keys_of(r)
        ex = _oom_excess(r, prof.mem_capacity)
        t = int(np.argmin(keys))  # the lowest index among equals
        if int(keys[t]) >= _key(perf):
            break
        dims = cand[t]
        perf = perf_of(int(r["info"][t]), r["iter"][t], r["max_mem"][t])
        stats["switched"].append(int(differs[t]))
    return dims, perf, stats
