"""ctypes declarations of libaceso.so (include/aceso.h). Argument marshalling only."""
import ctypes
import os

from .buildlib import LIB

c_i32, c_i64, c_u32, c_u64, c_sz, P = (ctypes.c_int32, ctypes.c_int64, ctypes.c_uint32,
                                        ctypes.c_uint64, ctypes.c_size_t, ctypes.c_void_p)

ACESO_OK, ACESO_EINVAL, ACESO_ERANGE, ACESO_ECUDA, ACESO_ENOMEM, ACESO_ENODEV = 0, -1, -2, -3, -4, -5
OUT_SUMMARY, OUT_FULL, FUSED_SELECT, HINT_DENSE, HINT_OVERLAP, PIPE_LITERAL = 1, 2, 4, 8, 16, 32
INFO_OOM = 1 << 16
INFO_INVALID = 1 << 17

SYMBOLS = ["aceso_load_profile", "aceso_free", "aceso_tiled_bytes", "aceso_pack_rowmajor",
           "aceso_select_buf_bytes", "aceso_eval", "aceso_select", "aceso_decode_key",
           "aceso_last_error", "aceso_version", "aceso_hash", "aceso_visited_bytes", "aceso_dedup", "aceso_expand",
           "aceso_enum_cuts_count", "aceso_enum_cuts", "aceso_schedule_name", "aceso_dims_bytes",
           "aceso_pack_dims", "aceso_eval_dims", "aceso_eval_global"]


class ProfileDesc(ctypes.Structure):
    _fields_ = [("n_ops", c_i32), ("n_types", c_i32), ("n_tp", c_i32), ("n_dp", c_i32),
                ("n_b", c_i32), ("n_devices", c_i32), ("op_type", P), ("rec", P), ("wmem", P),
                ("dps", P), ("mem_capacity", c_i64), ("global_batch", c_i64), ("rec_alt", P)]


class EvalOut(ctypes.Structure):
    _fields_ = [("iter_ns", P), ("max_mem", P), ("info", P), ("stage_T", P), ("stage_mem", P),
                ("stage_comp", P), ("stage_comm", P), ("p_max", c_i32)]


class SelectResult(ctypes.Structure):
    _fields_ = [("key", c_i64), ("cls_cost", c_u64), ("index", c_i64), ("reserved", c_u64)]


_lib = None


def load():
    """Loads the in-tree libaceso.so. Raises if it is missing: there is no fallback."""
    global _lib
    if _lib is not None:
        return _lib
    path = os.environ.get("ACESO_LIB_PATH") or LIB  # measurement knob: an alternative build
    if not os.path.exists(path):
        raise ImportError(f"libaceso.so not built ({path}); run __graft_entry__.build()")
    lib = ctypes.CDLL(path)
    lib.aceso_load_profile.argtypes = [ctypes.POINTER(ProfileDesc), ctypes.c_int, ctypes.POINTER(P)]
    lib.aceso_load_profile.restype = ctypes.c_int
    lib.aceso_free.argtypes = [P]
    lib.aceso_free.restype = None
    lib.aceso_tiled_bytes.argtypes = [c_i64, c_i32]
    lib.aceso_tiled_bytes.restype = c_sz
    lib.aceso_pack_rowmajor.argtypes = [P, c_i64, c_i32, P, P]
    lib.aceso_pack_rowmajor.restype = ctypes.c_int
    lib.aceso_select_buf_bytes.argtypes = [P, c_i64]
    lib.aceso_select_buf_bytes.restype = c_sz
    lib.aceso_eval.argtypes = [P, P, P, c_i64, c_i64, c_i64, c_u32, ctypes.POINTER(EvalOut), P, P]
    lib.aceso_eval.restype = ctypes.c_int
    lib.aceso_select.argtypes = [P, ctypes.POINTER(EvalOut), c_i64, c_i64, c_i64, P, P]
    lib.aceso_select.restype = ctypes.c_int
    lib.aceso_decode_key.argtypes = [c_i64, c_i64, ctypes.POINTER(ctypes.c_int),
                                     ctypes.POINTER(c_u64), ctypes.POINTER(c_i64),
                                     ctypes.POINTER(ctypes.c_int)]
    lib.aceso_decode_key.restype = ctypes.c_int
    lib.aceso_last_error.argtypes = []
    lib.aceso_last_error.restype = ctypes.c_char_p
    lib.aceso_version.argtypes = []
    lib.aceso_version.restype = ctypes.c_char_p
    lib.aceso_schedule_name.argtypes = [P, c_u32]
    lib.aceso_schedule_name.restype = ctypes.c_char_p
    lib.aceso_dims_bytes.argtypes = [c_i64, c_i32]
    lib.aceso_dims_bytes.restype = c_sz
    lib.aceso_pack_dims.argtypes = [P, c_i64, c_i32, P, P]
    lib.aceso_pack_dims.restype = ctypes.c_int
    lib.aceso_eval_dims.argtypes = [P, P, P, P, c_i64, c_i64, c_i64, c_u32, ctypes.POINTER(EvalOut), P, P]
    lib.aceso_eval_dims.restype = ctypes.c_int
    lib.aceso_eval_global.argtypes = [P, P, P, c_i64, c_i64, c_i64, c_u32, ctypes.POINTER(EvalOut), P, P, P]
    lib.aceso_eval_global.restype = ctypes.c_int
    lib.aceso_hash.argtypes = [P, P, c_i64, c_i32, P, P]
    lib.aceso_hash.restype = ctypes.c_int
    lib.aceso_visited_bytes.argtypes = [c_i64]
    lib.aceso_visited_bytes.restype = c_sz
    lib.aceso_dedup.argtypes = [P, c_i64, c_u32, P, c_i64, P, P, P]
    lib.aceso_dedup.restype = ctypes.c_int
    lib.aceso_expand.argtypes = [P, P, c_i32, c_i32, P, c_i64, P, P, P]
    lib.aceso_expand.restype = ctypes.c_int
    lib.aceso_enum_cuts_count.argtypes = [c_i32, c_i32]
    lib.aceso_enum_cuts_count.restype = c_i64
    lib.aceso_enum_cuts.argtypes = [c_i32, c_i32, ctypes.c_uint8, ctypes.c_uint64, c_i64, c_i64, P, P, P]
    lib.aceso_enum_cuts.restype = ctypes.c_int
    _lib = lib
    return lib
