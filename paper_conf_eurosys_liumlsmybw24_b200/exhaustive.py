"""Exp#4 baseline: the paper compares its search with a
dynamic-programming solver that explores a pruned configuration space with the same
performance model (10^7 - 4.3*10^7 configurations for GPT-3 2.6B / 6.7B). Here the pruned
space is enumerated exhaustively on the device and evaluated by aceso_eval, which returns the
space's exact optimum (what the DP solves for):

  stage-uniform configurations -- p pipeline stages (p a power of two, C(L-1, p-1) cut
  subsets at op granularity, up to `max_per_family`), every stage on G/p devices with the
  same (tp, dp), recomputation of all ops or none, every microbatch size whose per-GPU batch
  is in the profile.

The host only enumerates families (p, code, header); aceso_enum_cuts writes the candidates
of a family straight into the tiled layout, aceso_eval (SUMMARY + fused select) evaluates
them, and the exact (class<<62 | cost, index) pair of every batch is folded on the device.
"""
from __future__ import annotations

import math
import time

import numpy as np
import torch

from .api import Context, enum_cuts, enum_cuts_count
from .search import encode, header, perf_of


def families(prof, max_per_family: int = 1 << 27):
    """(p, code, hdr, count) of the pruned stage-uniform space."""
    L, G = prof.n_ops, prof.n_devices
    out = []
    p = 1
    while p <= min(G, L, 8):
        cnt = enum_cuts_count(L, p)
        if 0 <= cnt <= max_per_family and G % p == 0:
            g = int(math.log2(G // p))
            for tpl in range(0, min(g, prof.n_tp - 1) + 1):
                dpl = g - tpl
                if dpl >= prof.n_dp:
                    continue
                for rc in (0, 1):
                    code = encode(0, tpl, dpl, rc)
                    for mbs in range(dpl, dpl + prof.n_b):
                        if (1 << mbs) > prof.global_batch or prof.global_batch % (1 << mbs):
                            continue
                        out.append((p, code, int(header(mbs, p)), cnt))
        p *= 2
    return out


def colex_unrank(r: int, k: int):
    """The r-th k-subset of {0, 1, ...} in colex order (ascending)."""
    cut = []
    for i in range(k, 0, -1):
        x = i - 1
        while math.comb(x + 1, i) <= r:
            x += 1
        r -= math.comb(x, i)
        cut.append(x)
    return cut[::-1]


def configuration(prof, fam, r: int):
    """Row-major codes and header of candidate r of family fam."""
    p, code, hdr, _ = fam
    row = np.full(prof.n_ops, code & 0xFE, np.uint8)
    row[0] |= 1
    for c in colex_unrank(r, p - 1):
        row[c + 1] |= 1
    return row, np.uint64(hdr)


def exhaustive_best(prof, ctx: Context, batch: int = 1 << 22, max_per_family: int = 1 << 27):
    """Evaluates the whole pruned space; returns a dict with the optimum and the cost."""
    fams = families(prof, max_per_family)
    n_total = sum(f[3] for f in fams)
    dev = torch.device("cuda", ctx.device)
    cap = min(batch, max(f[3] for f in fams))
    tiled = ctx.alloc_tiled(cap)
    hd = torch.empty(cap, dtype=torch.int64, device=dev)
    out = ctx.alloc_outputs(cap)
    sel = ctx.alloc_select(cap)
    best = torch.tensor([(1 << 63) - 1, (1 << 63) - 1], dtype=torch.int64, device=dev)  # (cls_cost, index)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    off = 0
    launches = 0
    for fam in fams:
        p, code, hdr, cnt = fam
        for first in range(0, cnt, cap):
            n = min(cap, cnt - first)
            enum_cuts(prof.n_ops, p, code, hdr, first, n, tiled, hd)
            ctx.eval(tiled, hd, n=n, global_offset=off + first, n_total=n_total, summary=True, select=True,
                     out=out, sel=sel)
            pair = sel[8:24].view(torch.int64)  # exact (cls << 62 | cost, global index); index -1: none
            ok = pair[1] >= 0
            less = ok & ((pair[0] < best[0]) | ((pair[0] == best[0]) & (pair[1] < best[1])))
            best = torch.where(less, pair, best)
            launches += 2
        off += cnt
    torch.cuda.synchronize()
    dt = time.perf_counter() - t0
    cc, idx = int(best[0]), int(best[1])
    res = {"explored": n_total, "families": len(fams), "time_s": dt, "configs_per_s": n_total / dt,
           "gpu_launches": launches}
    if idx == (1 << 63) - 1:
        res["best"] = None
        return res
    acc = 0
    for fam in fams:
        if idx < acc + fam[3]:
            row, h = configuration(prof, fam, idx - acc)
            res["best"] = {"class": cc >> 62, "cost": cc & ((1 << 62) - 1), "index": idx, "p": fam[0],
                           "mbs_log2": int(h & np.uint64(0xFF)), "code": fam[1],
                           "cuts": [int(j) for j in np.nonzero(row & 1)[0][1:]]}
            res["codes"], res["hdr"] = row, h
            break
        acc += fam[3]
    return res


def megatron_grid(prof):
    """The paper's Megatron-LM baseline configuration space ("a grid search over
    all these options using ACESO's performance model"): global settings only -- p pipeline
    stages (p a power of two dividing the device count), every stage on G/p devices with the
    same (tp, dp), the ops partitioned evenly (stage i = ops [L i / p, L (i + 1) / p), the
    search's initial partition), recomputation of every op or none, every microbatch size whose
    per-GPU batch is in the profile. Returns row-major codes [n][L] and headers [n]."""
    L, G = prof.n_ops, prof.n_devices
    rows, hdrs = [], []
    p = 1
    while p <= min(G, L):
        if G % p == 0:
            g = int(math.log2(G // p))
            starts = [L * i // p for i in range(p)]
            for tpl in range(0, min(g, prof.n_tp - 1) + 1):
                dpl = g - tpl
                if dpl >= prof.n_dp:
                    continue
                for rc in (0, 1):
                    row = np.full(L, encode(0, tpl, dpl, rc), np.uint8)
                    row[starts] |= 1
                    for mbs in range(dpl, dpl + prof.n_b):
                        if (1 << mbs) > prof.global_batch or prof.global_batch % (1 << mbs):
                            continue
                        rows.append(row)
                        hdrs.append(header(mbs, p))
        p *= 2
    if not rows:
        return np.zeros((0, L), np.uint8), np.zeros(0, np.uint64)
    return np.stack(rows), np.array(hdrs, np.uint64)


def megatron_best(prof, evaluator):
    """Evaluates the Megatron grid (one batch through `evaluator.evaluate`); the best
    configuration by (class, cost) with the lowest index on ties (R12)."""
    codes, hdr = megatron_grid(prof)
    if len(hdr) == 0:
        return {"explored": 0, "best": None}
    r = evaluator.evaluate(codes, hdr)
    best, bi = None, -1
    for i in range(len(hdr)):
        key = perf_of(int(r["info"][i]), r["iter"][i], r["max_mem"][i])
        if key[0] < 2 and (best is None or key < best):
            best, bi = key, i
    out = {"explored": int(len(hdr)), "best": None}
    if best is not None:
        out["best"] = {"class": best[0], "cost": best[1], "index": bi, "p": int(hdr[bi] >> np.uint64(8)),
                       "mbs_log2": int(hdr[bi] & np.uint64(0xFF)), "code": int(codes[bi][0] & 0xFE)}
    return out
