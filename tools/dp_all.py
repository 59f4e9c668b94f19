"""Exp#4 on every BASELINE workload: exhaustive evaluation of the pruned
stage-uniform space (paper_conf_eurosys_liumlsmybw24_b200/exhaustive.py) next to the batched
search (search.py); one JSON line per workload."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_eurosys_liumlsmybw24_b200 as A  # noqa: E402
from aceso_inputs import profiles as P  # noqa: E402
from paper_conf_eurosys_liumlsmybw24_b200 import exhaustive as X  # noqa: E402
from paper_conf_eurosys_liumlsmybw24_b200 import search as S  # noqa: E402

budget = float(sys.argv[1]) if len(sys.argv) > 1 else 30.0
for name in ["toy-a", "toy-b", "gpt3-1.3b", "gpt3-13b", "t5", "wrn", "gpt-1k"]:
    prof = P.WORKLOADS[name]()
    ctx = A.Context(prof, 0)
    X.exhaustive_best(prof, ctx, max_per_family=1 << 10)  # warm-up
    dp = X.exhaustive_best(prof, ctx)
    codes, hdr = dp.pop("codes", None), dp.pop("hdr", None)
    kw = dict(budget_s=budget, patience=8)
    if name == "gpt-1k":
        kw.update(max_k=64, beam=2)
    res, st = S.search(prof, S.GPUEvaluator(ctx), **kw)
    line = {"workload": prof.name, "exhaustive": dp,
            "search": {"best": [res.perf[0], res.perf[1]], "explored": st["evaluated"], "time_s": st["time_s"]}}
    if codes is not None:  # hybrid: the search also starts from the exhaustive optimum
        hres, hst = S.search(prof, S.GPUEvaluator(ctx), starts=[(codes, int(hdr & 0xFF))], **kw)
        line["hybrid"] = {"best": [hres.perf[0], hres.perf[1]], "explored": hst["evaluated"] + dp["explored"],
                          "time_s": hst["time_s"] + dp["time_s"]}
    print(json.dumps(line), flush=True)
    ctx.close()
