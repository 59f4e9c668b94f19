"""Python binding of libaceso (same names as the C-ABI; argument marshalling only).

Every step of the evaluation path runs in the sm_100a kernels of libaceso.so;
PyTorch only provides device memory and streams. There is no CPU fallback: if
the library or a CUDA device is missing, these calls raise.

Unsigned 64-bit device arrays are carried in torch.int64 tensors (same bits);
`as_u64` / `as_u32` view them as numpy unsigned arrays on the host.
"""
from __future__ import annotations

import ctypes
import dataclasses

import numpy as np
import torch

from . import _lib as L


class AcesoError(RuntimeError):
    pass


def _check(rc, what):
    if rc != L.ACESO_OK:
        msg = L.load().aceso_last_error().decode()
        raise AcesoError(f"{what} failed ({rc}): {msg}")


def _ptr(t):
    return None if t is None else ctypes.c_void_p(t.data_ptr())


def _need(t, name, device, dtypes, numel):
    """Argument check before a pointer crosses the C-ABI: a host tensor, another device, a
    wrong element type or a short buffer would otherwise reach the kernel (a device fault)."""
    if not isinstance(t, torch.Tensor):
        raise TypeError(f"{name}: expected a torch.Tensor, got {type(t).__name__}")
    if t.device != device:  # the context's device (always a CUDA device outside tests)
        raise ValueError(f"{name}: must be on {device}, is on {t.device}")
    if t.dtype not in dtypes:
        raise ValueError(f"{name}: dtype {t.dtype} not in {dtypes}")
    if not t.is_contiguous():
        raise ValueError(f"{name}: must be contiguous")
    if t.numel() < numel:
        raise ValueError(f"{name}: {t.numel()} elements < {numel} needed")


_I64 = (torch.int64,)
_I32 = (torch.int32,)
_U8 = (torch.uint8,)


def _stream(stream):
    if stream is None:
        stream = torch.cuda.current_stream()
    return ctypes.c_void_p(stream.cuda_stream)


def version():
    return L.load().aceso_version().decode()


def tiled_bytes(n, n_ops):
    return int(L.load().aceso_tiled_bytes(int(n), int(n_ops)))


def as_u64(t):
    return t.detach().cpu().numpy().view(np.uint64)


def as_u32(t):
    return t.detach().cpu().numpy().view(np.uint32)


@dataclasses.dataclass
class Outputs:
    """Device output arrays of one batch (SoA). Stage arrays are [p_max, n]."""
    iter_ns: torch.Tensor
    max_mem: torch.Tensor
    info: torch.Tensor
    stage_T: torch.Tensor | None = None
    stage_mem: torch.Tensor | None = None
    stage_comp: torch.Tensor | None = None
    stage_comm: torch.Tensor | None = None
    p_max: int = 0

    def c_struct(self):
        return L.EvalOut(_ptr(self.iter_ns), _ptr(self.max_mem), _ptr(self.info), _ptr(self.stage_T),
                         _ptr(self.stage_mem), _ptr(self.stage_comp), _ptr(self.stage_comm),
                         int(self.p_max))


@dataclasses.dataclass
class Selection:
    cls: int          # 0 feasible, 1 OOM, -1 nothing valid
    cost: int         # iteration time (cls 0) or max stage memory (cls 1)
    index: int        # global candidate index, -1 if nothing valid
    key: int          # packed all-reduce key

    @classmethod
    def from_buffer(cls, sel: torch.Tensor):
        raw = sel[:32].cpu().numpy()
        key = int(raw[0:8].view(np.int64)[0])
        cc = int(raw[8:16].view(np.uint64)[0])
        idx = int(raw[16:24].view(np.int64)[0])
        if idx < 0:
            return cls(-1, 0, -1, key)
        return cls(cc >> 62, cc & ((1 << 62) - 1), idx, key)


class Context:
    """aceso_load_profile / aceso_free: a packed, device-resident op-cost profile."""

    def __init__(self, profile, device: int = 0):
        lib = L.load()
        self.device = int(device)
        self.profile = profile
        alt = getattr(profile, "rec_alt", None)
        self._keep = [np.ascontiguousarray(profile.op_type, dtype=np.uint16),
                      np.ascontiguousarray(profile.rec, dtype=np.int64),
                      np.ascontiguousarray(profile.wmem, dtype=np.int64),
                      np.ascontiguousarray(profile.dps, dtype=np.int64),
                      None if alt is None else np.ascontiguousarray(alt, dtype=np.int64)]
        ot, rec, wm, dps, ra = self._keep
        desc = L.ProfileDesc(int(ot.shape[0]), int(rec.shape[0]), int(rec.shape[1]), int(dps.shape[2]),
                             int(rec.shape[2]), int(profile.n_devices), ot.ctypes.data, rec.ctypes.data,
                             wm.ctypes.data, dps.ctypes.data, int(profile.mem_capacity),
                             int(profile.global_batch), None if ra is None else ra.ctypes.data)
        h = ctypes.c_void_p()
        _check(lib.aceso_load_profile(ctypes.byref(desc), self.device, ctypes.byref(h)),
               "aceso_load_profile")
        self._h = h
        self.n_ops = int(ot.shape[0])
        self.n_devices = int(profile.n_devices)
        self._dev = torch.device("cuda", self.device)

    def close(self):
        if getattr(self, "_h", None):
            L.load().aceso_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def schedule(self, dense_hint: bool = False) -> str:
        """aceso_schedule_name: the kernel aceso_eval runs on this context."""
        return L.load().aceso_schedule_name(self._h, L.HINT_DENSE if dense_hint else 0).decode()

    # -- buffers --------------------------------------------------------------
    def alloc_outputs(self, n: int, full: bool = False) -> Outputs:
        d = self._dev
        o = Outputs(torch.empty(n, dtype=torch.int64, device=d), torch.empty(n, dtype=torch.int64, device=d),
                    torch.empty(n, dtype=torch.int32, device=d))
        if full:
            pm = self.n_devices
            o.p_max = pm
            o.stage_T = torch.zeros((pm, n), dtype=torch.int64, device=d)
            o.stage_mem = torch.zeros((pm, n), dtype=torch.int64, device=d)
            o.stage_comp = torch.zeros((pm, n), dtype=torch.int64, device=d)
            o.stage_comm = torch.zeros((pm, n), dtype=torch.int64, device=d)
        return o

    def _check_outputs(self, out: Outputs, n: int, summary: bool, full: bool):
        d = self._dev
        if summary and n > 0:
            _need(out.iter_ns, "out.iter_ns", d, _I64, n)
            _need(out.max_mem, "out.max_mem", d, _I64, n)
            _need(out.info, "out.info", d, _I32, n)
        if full and n > 0:
            for k in ("stage_T", "stage_mem", "stage_comp", "stage_comm"):
                _need(getattr(out, k), f"out.{k}", d, _I64, int(out.p_max) * n)

    def alloc_select(self, n: int = 0) -> torch.Tensor:
        nb = int(L.load().aceso_select_buf_bytes(self._h, int(n)))
        return torch.zeros(nb, dtype=torch.uint8, device=self._dev)

    def alloc_tiled(self, n: int) -> torch.Tensor:
        return torch.zeros(tiled_bytes(n, self.n_ops), dtype=torch.uint8, device=self._dev)

    # -- C-ABI calls ------------------------------------------------------------
    def pack_rowmajor(self, codes: torch.Tensor, tiled: torch.Tensor | None = None, stream=None):
        """aceso_pack_rowmajor: device row-major [n, L] uint8 -> tiled layout."""
        assert codes.is_cuda and codes.dtype == torch.uint8 and codes.dim() == 2
        n = int(codes.shape[0])
        if tiled is None:
            tiled = self.alloc_tiled(n)
        codes = codes.contiguous()
        _need(codes, "codes", self._dev, _U8, n * self.n_ops)
        _need(tiled, "tiled", self._dev, _U8, tiled_bytes(n, self.n_ops))
        _check(L.load().aceso_pack_rowmajor(_ptr(codes), n, int(codes.shape[1]), _ptr(tiled),
                                            _stream(stream)), "aceso_pack_rowmajor")
        return tiled

    def eval(self, codes: torch.Tensor, hdr: torch.Tensor, n: int | None = None, global_offset: int = 0,
             n_total: int | None = None, summary: bool = True, full: bool = False, select: bool = True,
             out: Outputs | None = None, sel: torch.Tensor | None = None, stream=None,
             dense_hint: bool = False, overlap_hint: bool = False, dims: torch.Tensor | None = None,
             literal: bool = False, global_key: int | torch.Tensor | None = None):
        """aceso_eval on tiled device codes and int64 device headers.

        dense_hint sets ACESO_HINT_DENSE (per-op kernel; identical results).
        overlap_hint sets ACESO_HINT_OVERLAP (the caller overlaps independent batches on
        several streams: throughput launch geometry; identical results).
        dims: tiled dimension plane (aceso_eval_dims; pack_dims builds it): ops whose bit is set
        run under their alternative tensor-parallel partition dimension.
        global_key: int64 tensor element or raw device address (e.g. a peer-mapped symmetric-
        memory pointer): aceso_eval_global joins the batch's packed key into it (atomic MIN).
        Returns (out, sel): the output arrays (or None) and the select buffer (or None)."""
        n = int(hdr.shape[0]) if n is None else int(n)
        n_total = global_offset + n if n_total is None else int(n_total)
        flags = (L.OUT_SUMMARY if summary else 0) | (L.OUT_FULL if full else 0) | (L.FUSED_SELECT if select else 0)
        if dense_hint:
            flags |= L.HINT_DENSE
        if overlap_hint:
            flags |= L.HINT_OVERLAP
        if literal:
            flags |= L.PIPE_LITERAL  # Eq. 2 as printed (R1 variant)
        if (summary or full) and out is None:
            out = self.alloc_outputs(n, full=full)
        if select and sel is None:
            sel = self.alloc_select(n)
        d = self._dev
        if n > 0:
            _need(codes, "codes", d, _U8, tiled_bytes(n, self.n_ops))
            _need(hdr, "hdr", d, _I64, n)
        if out is not None:
            self._check_outputs(out, n, summary, full)
        if select:
            _need(sel, "sel", d, _U8, int(L.load().aceso_select_buf_bytes(self._h, n)))
        if dims is not None and n > 0:
            _need(dims, "dims", d, _U8, int(L.load().aceso_dims_bytes(n, self.n_ops)))
        cs = out.c_struct() if out is not None else None
        if global_key is not None:
            assert dims is None and select
            gk = global_key.data_ptr() if isinstance(global_key, torch.Tensor) else int(global_key)
            rc = L.load().aceso_eval_global(self._h, _ptr(codes), _ptr(hdr), n, int(global_offset), n_total, flags,
                                            ctypes.byref(cs) if cs is not None else None, _ptr(sel),
                                            ctypes.c_void_p(gk), _stream(stream))
            _check(rc, "aceso_eval_global")
            return out, sel
        if dims is not None:
            rc = L.load().aceso_eval_dims(self._h, _ptr(codes), _ptr(dims), _ptr(hdr), n, int(global_offset), n_total,
                                          flags, ctypes.byref(cs) if cs is not None else None, _ptr(sel),
                                          _stream(stream))
            _check(rc, "aceso_eval_dims")
            return out, sel
        rc = L.load().aceso_eval(self._h, _ptr(codes), _ptr(hdr), n, int(global_offset), n_total, flags,
                                 ctypes.byref(cs) if cs is not None else None, _ptr(sel), _stream(stream))
        _check(rc, "aceso_eval")
        return out, sel

    def pack_dims(self, dims: torch.Tensor, plane: torch.Tensor | None = None, stream=None):
        """aceso_pack_dims: device row-major [n, L] uint8 (nonzero = alternative dimension) ->
        tiled dimension plane."""
        assert dims.is_cuda and dims.dtype == torch.uint8 and dims.dim() == 2
        n = int(dims.shape[0])
        if plane is None:
            plane = torch.zeros(max(2, int(L.load().aceso_dims_bytes(n, self.n_ops))), dtype=torch.uint8,
                                device=self._dev)
        dims = dims.contiguous()
        _need(plane, "plane", self._dev, _U8, int(L.load().aceso_dims_bytes(n, self.n_ops)))
        _check(L.load().aceso_pack_dims(_ptr(dims), n, int(dims.shape[1]), _ptr(plane), _stream(stream)),
               "aceso_pack_dims")
        return plane

    def expand(self, bases: torch.Tensor, cands: torch.Tensor, ranks: torch.Tensor | None = None,
               n: int | None = None, tiled: torch.Tensor | None = None, hdr: torch.Tensor | None = None,
               stream=None):
        """aceso_expand: device candidates (base + patches, uint8 view of aceso_cand rows) ->
        (tiled codes, int64 headers)."""
        n = int(cands.numel() // 56) if n is None else int(n)
        if tiled is None:
            tiled = self.alloc_tiled(max(n, 1))
        if hdr is None:
            hdr = torch.empty(max(n, 1), dtype=torch.int64, device=self._dev)
        nb = int(bases.shape[0])
        d, stride = self._dev, 16 * ((self.n_ops + 15) // 16)
        if n > 0:
            _need(bases, "bases", d, _U8, nb * stride)
            _need(cands, "cands", d, _U8, 56 * n)
            if ranks is not None:
                _need(ranks, "ranks", d, (torch.int16,), nb * 2 * stride)
            _need(tiled, "tiled", d, _U8, tiled_bytes(n, self.n_ops))
            _need(hdr, "hdr", d, _I64, n)
        _check(L.load().aceso_expand(_ptr(bases), _ptr(ranks) if ranks is not None else None, nb,
                                     self.n_ops, _ptr(cands), n, _ptr(tiled), _ptr(hdr), _stream(stream)),
               "aceso_expand")
        return tiled, hdr[:n]

    def select(self, out: Outputs, n: int | None = None, global_offset: int = 0,
               n_total: int | None = None, sel: torch.Tensor | None = None, stream=None):
        """aceso_select: argmin over an already written summary."""
        n = int(out.iter_ns.shape[0]) if n is None else int(n)
        n_total = global_offset + n if n_total is None else int(n_total)
        if sel is None:
            sel = self.alloc_select(n)
        self._check_outputs(out, n, True, False)
        _need(sel, "sel", self._dev, _U8, int(L.load().aceso_select_buf_bytes(self._h, n)))
        cs = out.c_struct()
        _check(L.load().aceso_select(self._h, ctypes.byref(cs), n, int(global_offset), n_total, _ptr(sel),
                                     _stream(stream)), "aceso_select")
        return sel


def hash_candidates(codes: torch.Tensor, hdr: torch.Tensor, n_ops: int, n: int | None = None,
                    out: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """aceso_hash: 64-bit configuration hash of every candidate of a tiled batch (int64 view)."""
    n = int(hdr.shape[0]) if n is None else int(n)
    if out is None:
        out = torch.empty(n, dtype=torch.int64, device=hdr.device)
    if n > 0:
        d = hdr.device
        _need(codes, "codes", d, _U8, tiled_bytes(n, n_ops))
        _need(hdr, "hdr", d, _I64, n)
        _need(out, "out", d, _I64, n)
    _check(L.load().aceso_hash(_ptr(codes), _ptr(hdr), n, int(n_ops), _ptr(out), _stream(stream)),
           "aceso_hash")
    return out


class VisitedSet:
    """Device visited set of configuration hashes (aceso_dedup): first occurrence across calls."""

    def __init__(self, slots: int, device: int = 0):
        nb = int(L.load().aceso_visited_bytes(int(slots)))
        if nb == 0:
            raise AcesoError("slots must be a power of two >= 2")
        self.slots = int(slots)
        self.table = torch.zeros(nb, dtype=torch.uint8, device=torch.device("cuda", device))
        self.status = torch.zeros(1, dtype=torch.int32, device=self.table.device)
        self.epoch = 0

    def insert(self, hashes: torch.Tensor, dup: torch.Tensor | None = None, stream=None) -> torch.Tensor:
        """Marks dup[i] = 1 for hashes seen in an earlier call or at a lower index of this one."""
        n = int(hashes.shape[0])
        if dup is None:
            dup = torch.empty(n, dtype=torch.uint8, device=hashes.device)
        d = self.table.device
        if n > 0:
            _need(hashes, "hashes", d, _I64, n)
            _need(dup, "dup", d, _U8, n)
        self.epoch += 1
        _check(L.load().aceso_dedup(_ptr(hashes), n, self.epoch, _ptr(self.table), self.slots, _ptr(dup),
                                    _ptr(self.status), _stream(stream)), "aceso_dedup")
        return dup

    def overflowed(self) -> bool:
        return bool(self.status.item())


def decode_key(key: int, n_total: int):
    """aceso_decode_key -> (cls, cost, index, saturated)."""
    cls = ctypes.c_int()
    cost = ctypes.c_uint64()
    idx = ctypes.c_int64()
    sat = ctypes.c_int()
    _check(L.load().aceso_decode_key(int(key), int(n_total), ctypes.byref(cls), ctypes.byref(cost),
                                     ctypes.byref(idx), ctypes.byref(sat)), "aceso_decode_key")
    return cls.value, cost.value, idx.value, bool(sat.value)


def enum_cuts_count(n_ops: int, p: int) -> int:
    """aceso_enum_cuts_count: C(n_ops - 1, p - 1), or -1 outside the supported range."""
    return int(L.load().aceso_enum_cuts_count(int(n_ops), int(p)))


def enum_cuts(n_ops: int, p: int, code: int, hdr: int, first: int, n: int, tiled: torch.Tensor,
              hdr_out: torch.Tensor, stream=None):
    """aceso_enum_cuts: candidates [first, first + n) of the stage-partition family (p, code,
    hdr) written to device `tiled` (uint8, tiled layout) and `hdr_out` (int64)."""
    if n > 0:
        d = tiled.device
        _need(tiled, "tiled", d, _U8, tiled_bytes(n, n_ops))
        _need(hdr_out, "hdr_out", d, _I64, n)
    _check(L.load().aceso_enum_cuts(int(n_ops), int(p), int(code) & 0xFF, int(hdr), int(first), int(n),
                                    _ptr(tiled), _ptr(hdr_out), _stream(stream)), "aceso_enum_cuts")


def upload_candidates(codes_tiled: np.ndarray, hdr: np.ndarray, device=0, pin=False):
    """Host tiled codes + uint64 headers -> device tensors (tiled uint8, int64 headers)."""
    c = torch.from_numpy(np.ascontiguousarray(codes_tiled, dtype=np.uint8))
    h = torch.from_numpy(np.ascontiguousarray(hdr, dtype=np.uint64).view(np.int64))
    if pin:
        c, h = c.pin_memory(), h.pin_memory()
    dev = torch.device("cuda", device)
    return c.to(dev, non_blocking=pin), h.to(dev, non_blocking=pin)
