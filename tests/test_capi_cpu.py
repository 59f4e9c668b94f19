"""C-ABI library checks that need no GPU: the library loads, exports every symbol
that include/aceso.h declares, validates profiles before touching a device, and
decodes keys. (Compute calls need a GPU: see test_gpu_parity.py.)"""
import ctypes
import os
import re

import numpy as np
import pytest

import aceso_inputs as ai
from aceso_inputs import profiles as P
from paper_conf_eurosys_liumlsmybw24_b200 import _lib as L
from paper_conf_eurosys_liumlsmybw24_b200 import api

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_functions():
    txt = open(os.path.join(ROOT, "include", "aceso.h")).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(aceso_[a-z_]+)\s*\(", txt)))


def test_library_exports_every_declared_symbol():
    lib = L.load()
    names = header_functions()
    assert set(names) == set(L.SYMBOLS), names
    for name in names:
        assert hasattr(lib, name), name
    # exported with C linkage (no mangling)
    out = os.popen(f"nm -D --defined-only {L.LIB}").read()
    for name in names:
        assert re.search(rf"\bT {name}\b", out), name


def test_library_is_sm100a():
    out = os.popen(f"/usr/local/cuda/bin/cuobjdump -lelf {L.LIB} 2>&1").read()
    assert "sm_100a" in out


def test_tiled_bytes():
    assert api.tiled_bytes(0, 5) == 0
    assert api.tiled_bytes(1, 1) == 512
    assert api.tiled_bytes(33, 16) == 1024
    assert api.tiled_bytes(64, 17) == 2 * 2 * 512


def test_decode_key_roundtrip():
    for n_total in [1, 2, 1000, 65536, 1 << 20, (1 << 23) + 5]:
        ib = max(1, n_total.bit_length())
        cmax = (1 << (62 - ib)) - 1
        for cls in (0, 1):
            for cost in (0, 1, 12345, cmax - 1):
                for idx in (0, n_total - 1):
                    key = (cls << 62) | (cost << ib) | idx
                    assert api.decode_key(key, n_total) == (cls, cost, idx, False)
            key = (cls << 62) | (cmax << ib) | min(7, n_total - 1)
            assert api.decode_key(key, n_total)[3] is True
    assert api.decode_key((1 << 63) - 1, 10) == (-1, 0, -1, False)


def _desc(prof):
    keep = [np.ascontiguousarray(prof.op_type, np.uint16), np.ascontiguousarray(prof.rec, np.int64),
            np.ascontiguousarray(prof.wmem, np.int64), np.ascontiguousarray(prof.dps, np.int64)]
    d = L.ProfileDesc(prof.n_ops, prof.n_types, prof.n_tp, prof.n_dp, prof.n_b, prof.n_devices,
                      keep[0].ctypes.data, keep[1].ctypes.data, keep[2].ctypes.data, keep[3].ctypes.data,
                      prof.mem_capacity, prof.global_batch)
    return d, keep


def _load(prof):
    lib = L.load()
    d, keep = _desc(prof)
    h = ctypes.c_void_p()
    rc = lib.aceso_load_profile(ctypes.byref(d), 0, ctypes.byref(h))
    msg = lib.aceso_last_error().decode()
    if rc == 0:
        lib.aceso_free(h)
    return rc, msg


@pytest.mark.parametrize("mutate,code", [
    (lambda p: p.rec.__setitem__((0, 0, 0, 5), p.rec[0, 0, 0, 4] + 1), L.ACESO_ERANGE),   # keep > act
    (lambda p: p.rec.__setitem__((0, 0, 0, 0), 1 << 32), L.ACESO_ERANGE),               # > u32
    (lambda p: p.rec.__setitem__((0, 0, 0, 2), -1), L.ACESO_ERANGE),                    # negative
    (lambda p: p.wmem.__setitem__((0, 0, 0), (1 << 40) + 1), L.ACESO_ERANGE),           # W > 2^40
    (lambda p: p.rec.__setitem__((0, 0, 0, 6), (1 << 40) + 1), L.ACESO_ERANGE),         # peak > 2^40
    # wide but valid memory values are accepted (served by the exact 64-bit scan kernel); on a
    # box without a GPU the load then stops at the device probe
    (lambda p: p.wmem.__setitem__((0, 0, 0), (1 << 40) - 1), L.ACESO_ENODEV),
    (lambda p: p.rec.__setitem__((0, 0, 0, 4), (1 << 39) + 1), L.ACESO_ENODEV),
    (lambda p: p.op_type.__setitem__(0, 999), L.ACESO_EINVAL),                          # bad type
    (lambda p: setattr(p, "global_batch", 0), L.ACESO_EINVAL),
    (lambda p: setattr(p, "n_devices", 256), L.ACESO_EINVAL),
])
def test_profile_validation_before_device(mutate, code):
    prof = P.toy_a()
    mutate(prof)
    rc, msg = _load(prof)
    assert rc == code and msg


def test_valid_profile_reaches_device_probe():
    import torch
    rc, msg = _load(P.toy_a())
    if torch.cuda.is_available():
        assert rc == 0, msg
    else:
        assert rc in (L.ACESO_ENODEV, L.ACESO_ECUDA) and msg


def test_eval_rejects_bad_arguments():
    lib = L.load()
    rc = lib.aceso_eval(None, None, None, 0, 0, 0, 1, None, None, None)
    assert rc == L.ACESO_EINVAL


def test_every_workload_profile_is_accepted_by_validation():
    """All BASELINE.json workloads pass the range rules (they stop only at the device probe)."""
    import torch
    for name, fn in P.WORKLOADS.items():
        rc, msg = _load(fn())
        assert rc == 0 or (not torch.cuda.is_available() and rc in (L.ACESO_ENODEV, L.ACESO_ECUDA)), (name, msg)


def test_dedup_rejects_bad_arguments():
    lib = L.load()
    assert lib.aceso_visited_bytes(1000) == 0 and lib.aceso_visited_bytes(1024) == 16 * 1024
    st = ctypes.c_uint32()
    # slots not a power of two / epoch 0 / epoch too large: rejected before any device call
    assert lib.aceso_dedup(None, 0, 1, ctypes.addressof(st), 1000, None, ctypes.addressof(st), None) == L.ACESO_EINVAL
    assert lib.aceso_dedup(None, 0, 0, ctypes.addressof(st), 1024, None, ctypes.addressof(st), None) == L.ACESO_EINVAL
    assert lib.aceso_dedup(None, 0, 1 << 23, ctypes.addressof(st), 1024, None, ctypes.addressof(st), None) == L.ACESO_EINVAL
    assert lib.aceso_hash(None, None, -1, 10, None, None) == L.ACESO_EINVAL


def test_hash_reference_is_order_and_header_sensitive():
    import sys
    sys.path.insert(0, os.path.dirname(__file__))
    from hash_reference import config_hash
    rng = np.random.default_rng(0)
    c = rng.integers(0, 256, size=(50, 37), dtype=np.uint8)
    h = rng.integers(0, 1 << 60, size=50, dtype=np.uint64)
    base = config_hash(c, h)
    assert len(set(base.tolist())) == 50
    c2 = c.copy()
    c2[:, [3, 4]] = c2[:, [4, 3]]
    assert (config_hash(c2, h) != base)[c[:, 3] != c[:, 4]].all()
    assert (config_hash(c, h ^ np.uint64(1 << 8)) != base).all()


def test_enum_cuts_count_is_the_binomial():
    import math
    from paper_conf_eurosys_liumlsmybw24_b200 import enum_cuts_count
    for L in (1, 6, 10, 315, 821, 13003, 16384):
        for p in range(1, 9):
            want = math.comb(L - 1, p - 1) if p <= L else -1
            got = enum_cuts_count(L, p)
            assert got == (want if 0 <= want < (1 << 62) else -1), (L, p, got, want)
    assert enum_cuts_count(315, 9) == -1 and enum_cuts_count(0, 1) == -1 and enum_cuts_count(315, 0) == -1


def test_binding_argument_checks_cpu():
    """The binding's tensor check (api._need) refuses a wrong device, dtype, a non-contiguous
    view and a short buffer before any pointer reaches the C-ABI (device = cpu stands in for
    the context's CUDA device here)."""
    import torch
    from paper_conf_eurosys_liumlsmybw24_b200.api import _need
    cpu = torch.device("cpu")
    t = torch.zeros(64, dtype=torch.int64)
    _need(t, "t", cpu, (torch.int64,), 64)  # passes
    with pytest.raises(ValueError):
        _need(t, "t", torch.device("cuda", 0), (torch.int64,), 64)
    with pytest.raises(ValueError):
        _need(t, "t", cpu, (torch.int32,), 64)
    with pytest.raises(ValueError):
        _need(t, "t", cpu, (torch.int64,), 65)
    with pytest.raises(ValueError):
        _need(t.view(8, 8).t(), "t", cpu, (torch.int64,), 8)
    with pytest.raises(TypeError):
        _need(t.numpy(), "t", cpu, (torch.int64,), 1)
