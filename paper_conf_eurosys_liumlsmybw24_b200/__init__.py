"""B200-native batched evaluator of Aceso's performance/memory model (EuroSys '24).

Public API (names follow include/aceso.h): Context (aceso_load_profile/aceso_free),
Context.eval (aceso_eval), Context.select (aceso_select), Context.pack_rowmajor
(aceso_pack_rowmajor), decode_key (aceso_decode_key), hash_candidates (aceso_hash),
VisitedSet (aceso_visited_bytes/aceso_dedup), enum_cuts / enum_cuts_count (aceso_enum_cuts,
the Exp#4 exhaustive baseline: exhaustive.py), dist.global_select (NCCL all-reduce MIN of the
packed key).
"""
from .api import AcesoError, Context, Outputs, Selection, VisitedSet, as_u32, as_u64, decode_key, \
    enum_cuts, enum_cuts_count, hash_candidates, tiled_bytes, upload_candidates, version  # noqa: F401
from .buildlib import LIB, build  # noqa: F401
