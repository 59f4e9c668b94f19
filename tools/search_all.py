"""Search time (batched Alg. 1/2 over aceso_eval) on every BASELINE workload; one JSON line each.
For the toy models the exhaustive optimum (aceso_eval over the whole space) is reported too."""
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import aceso_inputs as ai  # noqa: E402
import paper_conf_eurosys_liumlsmybw24_b200 as A  # noqa: E402
from aceso_inputs import profiles as P  # noqa: E402
from paper_conf_eurosys_liumlsmybw24_b200 import search as S  # noqa: E402
from paper_conf_eurosys_liumlsmybw24_b200.api import Selection  # noqa: E402

budget = float(sys.argv[1]) if len(sys.argv) > 1 else 60.0
for name in ["toy-a", "toy-b", "gpt3-1.3b", "gpt3-13b", "t5", "wrn", "gpt-1k"]:
    prof = P.WORKLOADS[name]()
    ctx = A.Context(prof, 0)
    ev = S.GPUEvaluator(ctx)
    kw = dict(budget_s=budget, patience=8)
    if name == "gpt-1k":
        kw.update(max_k=64, beam=2)
    t0 = time.perf_counter()
    res, st = S.search(prof, ev, **kw)
    line = {"workload": prof.name, "search_time_s": st["time_s"], "time_to_best_s": st["time_to_best_s"],
            "evaluated": st["evaluated"], "batches": st["batches"], "improvements": st["improvements"],
            "best": {"class": res.perf[0], "cost": res.perf[1], "p": int((res.codes & 1).sum()),
                     "mbs_log2": res.mbs}}
    inits = []
    for p in [1, 2, 4, 8, 16, 32, 64]:
        r0 = S.initial_config(prof, p) if p <= prof.n_devices else None
        if r0 is not None:
            o = ev.evaluate(r0[0][None, :], np.array([S.header(r0[1], p)], np.uint64))
            inits.append(S.perf_of(int(o["info"][0]), o["iter"][0], o["max_mem"][0]))
    line["initial_best"] = {"class": min(inits)[0], "cost": min(inits)[1]}
    if name in ("toy-a", "toy-b"):
        codes, hdr = ai.exhaustive(prof, per_op=(name == "toy-a"))
        tiled = torch.from_numpy(ai.tile(codes)).cuda()
        hd = torch.from_numpy(hdr.view(np.int64)).cuda()
        _, sel = ctx.eval(tiled, hd, summary=False, select=True)
        s = Selection.from_buffer(sel)
        line["exhaustive_optimum"] = {"class": s.cls, "cost": s.cost, "space": int(len(hdr))}
        line["reached_optimum"] = bool(res.perf == (s.cls, s.cost))
    print(json.dumps(line), flush=True)
    ctx.close()
