"""One workload, one batch, a few aceso_eval launches (for ncu captures).
usage: python tools/prof_one.py [workload] [n] [launches]
(parity against the oracle is the job of tests/; this tool does not use it)"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import aceso_inputs as ai  # noqa: E402
from aceso_inputs import profiles as P  # noqa: E402
import paper_conf_eurosys_liumlsmybw24_b200 as A  # noqa: E402
from paper_conf_eurosys_liumlsmybw24_b200.api import Selection  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "gpt3-1.3b"
n = int(sys.argv[2]) if len(sys.argv) > 2 else 65536
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
prof = P.WORKLOADS[name]()
ctx = A.Context(prof, 0)
codes, hdr = ai.search_shaped(prof, 20240422, 0, n, group_size=1024, tiled=True)
cd, hd = A.upload_candidates(codes, hdr, 0)
out = ctx.alloc_outputs(n)
sel = ctx.alloc_select(n)
st = torch.cuda.current_stream()
ev = [torch.cuda.Event(enable_timing=True) for _ in range(2 * reps)]
for r in range(reps):
    ev[2 * r].record(st)
    ctx.eval(cd, hd, n=n, out=out, sel=sel, select=True, stream=st)
    ev[2 * r + 1].record(st)
torch.cuda.synchronize()
print(name, n, "us per launch:", [round(ev[2 * r].elapsed_time(ev[2 * r + 1]) * 1e3, 1) for r in range(reps)])
s = Selection.from_buffer(sel)
print("select", s)
