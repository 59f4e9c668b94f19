"""Candidates as base configuration + byte-range patches (include/aceso.h, aceso_cand):
the form every reconfiguration primitive of Table 1 takes in the search
driver. `expand_host` states the patch semantics in numpy (host materialisation of the few
configurations the search keeps, and CPU evaluators in tests); `aceso_expand` does the
same on the device for whole batches."""
from __future__ import annotations

import numpy as np

PATCH_NONE, PATCH_MASK, PATCH_ADD, PATCH_RANK_RC = 0, 1, 2, 3
MAX_PATCH = 6

PATCH_DTYPE = np.dtype([("a", "<u2"), ("b", "<u2"), ("kind", "u1"), ("v0", "u1"), ("v1", "u1"),
                        ("v2", "u1")])
CAND_DTYPE = np.dtype([("base", "<u4"), ("mbs", "u1"), ("p", "u1"), ("n_patch", "u1"),
                       ("reserved", "u1"), ("patch", PATCH_DTYPE, (MAX_PATCH,))])
assert PATCH_DTYPE.itemsize == 8 and CAND_DTYPE.itemsize == 56


def stride_of(n_ops: int) -> int:
    return 16 * ((n_ops + 15) // 16)


def mask(a, b, and_, or_):
    return (a, b, PATCH_MASK, and_ & 0xFF, or_ & 0xFF, 0)


def add(a, b, dt, dd):
    return (a, b, PATCH_ADD, dt & 0xFF, dd & 0xFF, 0)


def rank_rc(a, b, k, which, clear):
    return (a, b, PATCH_RANK_RC, k & 0xFF, (k >> 8) & 0xFF, (which & 1) | (2 if clear else 0))


def make(base: int, mbs: int, p: int, patches) -> np.ndarray:
    c = np.zeros((), CAND_DTYPE)
    c["base"], c["mbs"], c["p"], c["n_patch"] = base, mbs, p, len(patches)
    for i, pt in enumerate(patches):
        c["patch"][i] = pt
    return c


def expand_host(bases: np.ndarray, ranks: np.ndarray | None, cands: np.ndarray, n_ops: int):
    """bases [nb][stride] u8, ranks [nb][2][stride] u16, cands [n] CAND_DTYPE ->
    (codes [n][n_ops] u8, hdr [n] u64). Patches apply in order."""
    n = len(cands)
    codes = np.empty((n, n_ops), np.uint8)
    for i in range(n):
        c = cands[i]
        b = int(c["base"])
        row = bases[b, :n_ops].copy()
        for pt in c["patch"][: int(c["n_patch"])]:
            a, e = min(int(pt["a"]), n_ops), min(int(pt["b"]), n_ops)
            if e <= a:
                continue
            kind = int(pt["kind"])
            if kind == PATCH_MASK:
                row[a:e] = (row[a:e] & np.uint8(pt["v0"])) | np.uint8(pt["v1"])
            elif kind == PATCH_ADD:
                dt, dd = int(np.int8(pt["v0"])), int(np.int8(pt["v1"]))
                tp = ((row[a:e] >> 1) & 7).astype(np.int16) + dt
                dp = ((row[a:e] >> 5) & 7).astype(np.int16) + dd
                row[a:e] = (row[a:e] & 0x11) | ((tp.astype(np.uint8) & 7) << 1) | ((dp.astype(np.uint8) & 7) << 5)
            elif kind == PATCH_RANK_RC:
                k = int(pt["v0"]) | (int(pt["v1"]) << 8)
                sel = ranks[b, int(pt["v2"]) & 1, a:e] < k
                if int(pt["v2"]) & 2:
                    row[a:e][sel] &= 0xEF
                else:
                    row[a:e][sel] |= 0x10
        codes[i] = row
    hdr = cands["mbs"].astype(np.uint64) | (cands["p"].astype(np.uint64) << np.uint64(8))
    return codes, hdr
