"""CPU ORACLE — test infrastructure only (see oracle/aceso_oracle.c header).

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
reference legs may import this package. It never touches the CUDA library.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

INFO_OOM = 1 << 16
INFO_INVALID = 1 << 17


def build(force=False):
    src = os.path.join(_HERE, "aceso_oracle.c")
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O2", "-Wall", "-shared", "-fPIC", "-pthread", "-o", _LIB, src])
    return _LIB


def _load():
    global _lib
    if _lib is None:
        # ACESO_ORACLE_LIB: a mutant build of aceso_oracle.c (tests/test_oracle_mutations.py
        # checks that the pins reject every one of them)
        path = os.environ.get("ACESO_ORACLE_LIB")
        if not path:
            build()
            path = _LIB
        lib = ctypes.CDLL(path)
        P = ctypes.c_void_p
        i32, i64 = ctypes.c_int32, ctypes.c_int64
        lib.oracle_eval.argtypes = [i32, i32, i32, i32, i32, i32, P, P, P, P, P, i64, i64, P, P, P, i64,
                                    i32, P, P, P, P, P, P, P, ctypes.c_int, ctypes.c_int]
        lib.oracle_eval.restype = ctypes.c_int
        lib.oracle_select.argtypes = [P, P, P, i64, i64, P, P, P]
        _lib = lib
    return _lib


def _ptr(a):
    return None if a is None else a.ctypes.data


def evaluate(prof, codes, hdr, full=False, threads=1, dims=None, literal=False):
    """Evaluates row-major codes [n][L] with headers [n]; dims (optional, row-major [n][L],
    nonzero = the op's alternative tensor-parallel partition dimension) needs prof.rec_alt.

    Returns dict(iter, max_mem, info[, stage_T, stage_mem, stage_comp, stage_comm]);
    stage arrays are [n][G] (rows i >= p and rows of invalid candidates are 0).
    literal: Eq. 2 as printed (steady phase of N microbatches; reading R1 uses N - 1)."""
    lib = _load()
    codes = np.ascontiguousarray(codes, dtype=np.uint8)
    if dims is not None:
        dims = np.ascontiguousarray(dims, dtype=np.uint8)
        assert dims.shape == codes.shape
    rec_alt = getattr(prof, "rec_alt", None)
    rec_alt = None if rec_alt is None else np.ascontiguousarray(rec_alt, dtype=np.int64)
    hdr = np.ascontiguousarray(hdr, dtype=np.uint64)
    n = int(hdr.shape[0])
    L = int(prof.op_type.shape[0])
    assert codes.shape == (n, L), (codes.shape, n, L)
    op_type = np.ascontiguousarray(prof.op_type, dtype=np.uint16)
    rec = np.ascontiguousarray(prof.rec, dtype=np.int64)
    wmem = np.ascontiguousarray(prof.wmem, dtype=np.int64)
    dps = np.ascontiguousarray(prof.dps, dtype=np.int64)
    T, n_tp, n_b = rec.shape[0], rec.shape[1], rec.shape[2]
    n_dp = dps.shape[2]
    G = int(prof.n_devices)
    out = dict(iter=np.zeros(n, np.uint64), max_mem=np.zeros(n, np.uint64),
               info=np.zeros(n, np.uint32))
    st = [None] * 4
    if full:
        for k, name in enumerate(["stage_T", "stage_mem", "stage_comp", "stage_comm"]):
            out[name] = np.zeros((n, G), np.uint64)
            st[k] = out[name]
    rc = lib.oracle_eval(L, T, n_tp, n_dp, n_b, G, _ptr(op_type), _ptr(rec), _ptr(rec_alt), _ptr(wmem),
                         _ptr(dps), int(prof.mem_capacity), int(prof.global_batch), _ptr(codes), _ptr(dims),
                         _ptr(hdr), n,
                         G, _ptr(out["iter"]), _ptr(out["max_mem"]), _ptr(out["info"]),
                         _ptr(st[0]), _ptr(st[1]), _ptr(st[2]), _ptr(st[3]), int(threads),
                         int(bool(literal)))
    assert rc == 0
    return out


def select(out, global_offset=0):
    """(class, cost, global index) of the best candidate; index -1 if none valid."""
    lib = _load()
    it = np.ascontiguousarray(out["iter"], np.uint64)
    mm = np.ascontiguousarray(out["max_mem"], np.uint64)
    info = np.ascontiguousarray(out["info"], np.uint32)
    cls = ctypes.c_int()
    cost = ctypes.c_uint64()
    idx = ctypes.c_int64()
    lib.oracle_select(_ptr(it), _ptr(mm), _ptr(info), int(it.shape[0]), int(global_offset),
                      ctypes.byref(cls), ctypes.byref(cost), ctypes.byref(idx))
    return cls.value, cost.value, idx.value
