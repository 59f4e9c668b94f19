"""One workload's search on cuda:0 with chosen stage counts; prints the improvement history and
the final configuration's stages (start, end, tp log2, dp log2, recomputed ops)."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from aceso_inputs import profiles as P  # noqa: E402
from paper_conf_eurosys_liumlsmybw24_b200 import Context  # noqa: E402
from paper_conf_eurosys_liumlsmybw24_b200 import search as S  # noqa: E402

name, ps, budget = sys.argv[1], [int(x) for x in sys.argv[2].split(",")], float(sys.argv[3])
kw = eval(sys.argv[4]) if len(sys.argv) > 4 else {}
prof = P.WORKLOADS[name]()
ctx = Context(prof, 0)
t = time.perf_counter()
res, st = S.search(prof, S.GPUEvaluator(ctx), p_values=ps, budget_s=budget, **kw)
h, e = S.stages_of(res.codes)
print(json.dumps({"workload": name, "p_values": ps, "search": list(res.perf), "time_s": time.perf_counter() - t,
                  "evaluated": st["evaluated"], "batches": st["batches"], "mbs_log2": res.mbs,
                  "stages": [(int(a), int(b), int((res.codes[a] >> 1) & 7), int(res.codes[a] >> 5),
                              int(((res.codes[a:b] >> 4) & 1).sum())) for a, b in zip(h, e)],
                  "history": [(round(a, 3), list(b)) for a, b in st["history"]][-30:]}))
