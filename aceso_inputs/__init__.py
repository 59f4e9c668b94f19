"""Seeded synthetic inputs shared by the oracle tests and the CUDA tests/bench.

Holds none of the method's arithmetic: profile tables (profiles.py) and
configuration encodings (gen.c, counter-based RNG). See DESIGN.md §4.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

from .profiles import Profile, WORKLOADS, from_tables  # noqa: F401

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = os.path.join(_HERE, "libaceso_inputs.so")
_lib = None


def build(force=False):
    src = os.path.join(_HERE, "gen.c")
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O2", "-Wall", "-shared", "-fPIC", "-o", _LIB, src])
    return _LIB


class _Model(ctypes.Structure):
    _fields_ = [("L", ctypes.c_int32), ("n_tp", ctypes.c_int32), ("n_dp", ctypes.c_int32),
                ("n_b", ctypes.c_int32), ("G", ctypes.c_int32), ("Bg", ctypes.c_int64),
                ("rc_rank", ctypes.c_void_p)]


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        P = ctypes.c_void_p
        lib.gen_search_shaped.argtypes = [P, ctypes.c_uint64, ctypes.c_int64, ctypes.c_int64,
                                          ctypes.c_int32, ctypes.c_int32, P, ctypes.c_int, P]
        lib.gen_dense_random.argtypes = [P, ctypes.c_uint64, ctypes.c_int64, ctypes.c_int64, P,
                                         ctypes.c_int, P]
        lib.gen_exhaustive.argtypes = [P, ctypes.c_int, P, P, ctypes.c_int64]
        lib.gen_exhaustive.restype = ctypes.c_int64
        lib.gen_tile.argtypes = [P, ctypes.c_int64, ctypes.c_int32, P]
        _lib = lib
    return _lib


def _model(prof: Profile):
    rr = np.ascontiguousarray(prof.rc_rank())
    m = _Model(prof.n_ops, prof.n_tp, prof.n_dp, prof.n_b, prof.n_devices, prof.global_batch,
               rr.ctypes.data)
    return m, rr


def tiled_bytes(n, L):
    return ((n + 31) // 32) * ((L + 15) // 16) * 512


def _alloc(n, L, tiled):
    if tiled:
        return np.zeros(tiled_bytes(n, L), dtype=np.uint8)
    return np.zeros((n, L), dtype=np.uint8)


def _parts(n, threads):
    """Splits [0, n) into up to `threads` ranges aligned to 32 candidates (whole tiles)."""
    k = max(1, min(threads, (n + 31) // 32))
    tiles = (n + 31) // 32
    cuts = [min(n, 32 * (tiles * i // k)) for i in range(k + 1)]
    return [(a, b) for a, b in zip(cuts[:-1], cuts[1:]) if b > a]


def _run_parts(fn, n, threads):
    parts = _parts(n, threads)
    if len(parts) == 1:
        fn(*parts[0])
        return
    from concurrent.futures import ThreadPoolExecutor  # ctypes calls release the GIL
    with ThreadPoolExecutor(len(parts)) as ex:
        for f in [ex.submit(fn, a, b) for a, b in parts]:
            f.result()


def search_shaped(prof: Profile, seed: int, first: int, n: int, group_size: int = 1024,
                  invalid_permille: int = 20, tiled: bool = False, threads: int = 1):
    """Candidates [first, first+n) of the search-shaped distribution.
    The generator is counter-based, so `threads` > 1 only splits the work (same bytes)."""
    lib = _load()
    m, keep = _model(prof)
    codes = _alloc(n, prof.n_ops, tiled)
    hdr = np.zeros(n, dtype=np.uint64)
    row = tiled_bytes(32, prof.n_ops) // 32 if tiled else prof.n_ops  # bytes per candidate

    def part(a, b):
        rc = lib.gen_search_shaped(ctypes.byref(m), seed, first + a, b - a, group_size, invalid_permille,
                                   codes.ctypes.data + a * row, int(tiled), hdr.ctypes.data + 8 * a)
        assert rc == 0
    _run_parts(part, n, threads)
    return codes, hdr


def dense_random(prof: Profile, seed: int, first: int, n: int, tiled: bool = False, threads: int = 1):
    lib = _load()
    m, keep = _model(prof)
    codes = _alloc(n, prof.n_ops, tiled)
    hdr = np.zeros(n, dtype=np.uint64)
    row = tiled_bytes(32, prof.n_ops) // 32 if tiled else prof.n_ops

    def part(a, b):
        rc = lib.gen_dense_random(ctypes.byref(m), seed, first + a, b - a, codes.ctypes.data + a * row,
                                  int(tiled), hdr.ctypes.data + 8 * a)
        assert rc == 0
    _run_parts(part, n, threads)
    return codes, hdr


def exhaustive(prof: Profile, per_op: bool = True, count_only: bool = False):
    lib = _load()
    m, keep = _model(prof)
    cnt = lib.gen_exhaustive(ctypes.byref(m), int(per_op), None, None, 0)
    assert cnt >= 0
    if count_only:
        return cnt
    codes = np.zeros((cnt, prof.n_ops), dtype=np.uint8)
    hdr = np.zeros(cnt, dtype=np.uint64)
    lib.gen_exhaustive(ctypes.byref(m), int(per_op), codes.ctypes.data, hdr.ctypes.data, cnt)
    return codes, hdr


def tile(codes: np.ndarray):
    """Row-major [n][L] -> tiled layout bytes."""
    lib = _load()
    codes = np.ascontiguousarray(codes, dtype=np.uint8)
    n, L = codes.shape
    out = np.empty(tiled_bytes(n, L), dtype=np.uint8)
    lib.gen_tile(codes.ctypes.data, n, L, out.ctypes.data)
    return out


def dims_bytes(n, L):
    return ((n + 31) // 32) * ((L + 15) // 16) * 64


def tile_dims(dims: np.ndarray):
    """Row-major dimension bytes [n][L] (nonzero = alternative) -> the tiled plane
    (include/aceso.h: one little-endian u16 per candidate and 16-op chunk)."""
    dims = np.ascontiguousarray(dims != 0, dtype=np.uint8)
    n, L = dims.shape
    nch = (L + 15) // 16
    pad = np.zeros(((n + 31) // 32 * 32, nch * 16), np.uint8)
    pad[:n, :L] = dims
    bits = pad.reshape(-1, 32, nch, 16).astype(np.uint16) << np.arange(16, dtype=np.uint16)
    plane = bits.sum(axis=3, dtype=np.uint16).transpose(0, 2, 1)  # [tile][chunk][lane]
    return np.ascontiguousarray(plane).view(np.uint8).reshape(-1)


def code(head, tpl, dpl, rc):
    return (head & 1) | ((tpl & 7) << 1) | ((rc & 1) << 4) | ((dpl & 7) << 5)


def header(mbs_log2, p):
    return (mbs_log2 & 0xFF) | ((p & 0xFF) << 8)
