"""Small evaluation in the overlap-hint geometry (two tiles per warp, ragged last tile) for
compute-sanitizer (memcheck / racecheck / synccheck); checks the results against the oracle."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import aceso_inputs as ai
import oracle
from aceso_inputs import profiles as P
import paper_conf_eurosys_liumlsmybw24_b200 as A
from paper_conf_eurosys_liumlsmybw24_b200.api import Selection, as_u32, as_u64

prof = P.WORKLOADS["gpt3-1.3b"]()
n = 32 * 8 * 2 * 3 + 17  # 3 CTAs of 8 warps x 2 tiles, plus a ragged tile
codes, hdr = ai.search_shaped(prof, 20240422, 0, n, group_size=32)
ctx = A.Context(prof, 0)
tiled = torch.from_numpy(ai.tile(codes)).cuda()
hd = torch.from_numpy(hdr.view(np.int64)).cuda()
out, sel = ctx.eval(tiled, hd, select=True, overlap_hint=True)
torch.cuda.synchronize()
o = oracle.evaluate(prof, codes, hdr, threads=4)
assert np.array_equal(as_u64(out.iter_ns), o["iter"])
assert np.array_equal(as_u32(out.info), o["info"])
s = Selection.from_buffer(sel)
assert (s.cls, s.cost, s.index) == oracle.select(o)
print("overlap-hint sanitizer run ok:", n, "candidates")
