"""Small evaluations for compute-sanitizer (memcheck / racecheck / synccheck) on the round-2
paths: the scan kernel (wide memory values: u64 transient tables; and the u32 variant via
ACESO_KERNEL=scan), the dense kernel with a dimension plane (shared-memory and global tables),
ACESO_PIPE_LITERAL and the event kernel's two ring-slot sizes; every result checked against the
oracle."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import aceso_inputs as ai
import oracle
from aceso_inputs import profiles as P
import paper_conf_eurosys_liumlsmybw24_b200 as A
from paper_conf_eurosys_liumlsmybw24_b200.api import Selection, as_u32, as_u64


def check(prof, n, dims=False, literal=False, full=False):
    codes, hdr = ai.search_shaped(prof, 20240422, 0, n, group_size=32)
    d = (np.random.default_rng(1).random(codes.shape) < 0.3).astype(np.uint8) if dims else None
    ctx = A.Context(prof, 0)
    tiled = torch.from_numpy(ai.tile(codes)).cuda()
    hd = torch.from_numpy(hdr.view(np.int64)).cuda()
    plane = torch.from_numpy(ai.tile_dims(d)).cuda() if dims else None
    out, sel = ctx.eval(tiled, hd, select=True, full=full, dims=plane, literal=literal)
    torch.cuda.synchronize()
    o = oracle.evaluate(prof, codes, hdr, threads=4, dims=d, literal=literal)
    assert np.array_equal(as_u64(out.iter_ns), o["iter"]) and np.array_equal(as_u32(out.info), o["info"])
    s = Selection.from_buffer(sel)
    assert (s.cls, s.cost, s.index) == oracle.select(o)
    print(prof.name, ctx.schedule(), "dims" if dims else "", "literal" if literal else "", "ok", n)
    ctx.close()


n = 32 * 8 * 2 + 17  # two CTAs of 8 warps, plus a ragged tile
check(P.jittered(P.WORKLOADS["gpt3-1.3b"](), 5, 0, scale=64), n, full=True)   # scan kernel, E64
check(P.jittered(P.WORKLOADS["t5"](), 6, 3), 333)                            # event kernel
os.environ["ACESO_KERNEL"] = "scan"
check(P.WORKLOADS["gpt3-1.3b"](), n, literal=True)                            # scan kernel, E32
del os.environ["ACESO_KERNEL"]
check(P.WORKLOADS["gpt3-1.3b"](), n, dims=True, full=True)                    # dense + plane, smem tables
check(P.WORKLOADS["wrn"](), 200, dims=True)                                   # dense + plane, global tables
# event kernel with 8-chunk ring slots (2 CTAs per SM: SUMMARY + select) and 4-chunk slots
# (FULL), every warp walking two tiles through its ring
os.environ["ACESO_TILES_PER_WARP"] = "2"
check(P.WORKLOADS["gpt-1k"](), 32 * 3 + 5)
check(P.WORKLOADS["gpt-1k"](), 32 * 3 + 5, full=True)
del os.environ["ACESO_TILES_PER_WARP"]
print("round-2 sanitizer run ok")
