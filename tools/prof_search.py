import cProfile, pstats, sys, os, time
sys.path.insert(0, os.getcwd())
from aceso_inputs import profiles as P
from paper_conf_eurosys_liumlsmybw24_b200 import Context
from paper_conf_eurosys_liumlsmybw24_b200 import search as S
prof = P.WORKLOADS[sys.argv[1]]()
ctx = Context(prof, 0)
ev = S.GPUEvaluator(ctx)
S.search(prof, ev, budget_s=5, patience=8, max_batches=3)  # warm
pr = cProfile.Profile()
t = time.time()
pr.enable()
res, st = S.search(prof, ev, budget_s=20.0, patience=8)
pr.disable()
print("time", time.time() - t, res.perf, st["batches"], st["evaluated"])
pstats.Stats(pr).sort_stats("cumulative").print_stats(35)
