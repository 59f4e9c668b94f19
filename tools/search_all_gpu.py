"""Search on every BASELINE workload on cuda:0 (bench settings: 20 s budget, per-search patience
8) next to the Megatron grid and the Exp#4 stage-uniform optimum. One JSON line each."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

from aceso_inputs import profiles as P
from paper_conf_eurosys_liumlsmybw24_b200 import Context
from paper_conf_eurosys_liumlsmybw24_b200 import exhaustive as X
from paper_conf_eurosys_liumlsmybw24_b200 import search as S

names = sys.argv[1:] or ["toy-a", "toy-b", "gpt3-1.3b", "gpt3-13b", "t5", "wrn", "gpt-1k"]
for name in names:
    prof = P.WORKLOADS[name]()
    ctx = Context(prof, 0)
    ev = S.GPUEvaluator(ctx)
    t = time.perf_counter()
    res, st = S.search(prof, ev, budget_s=20.0, patience=8)
    dt = time.perf_counter() - t
    meg = X.megatron_best(prof, ev)
    h, e = S.stages_of(res.codes)
    print(json.dumps({"workload": name, "search": list(res.perf), "time_s": round(dt, 3),
                      "time_to_best_s": round(st["time_to_best_s"], 3), "evaluated": st["evaluated"],
                      "batches": st["batches"], "p": len(h), "mbs_log2": res.mbs,
                      "megatron_grid": [meg["best"]["class"], meg["best"]["cost"]] if meg["best"] else None}),
          flush=True)
    ctx.close()
