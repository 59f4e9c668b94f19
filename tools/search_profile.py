"""cProfile of the batched search driver on one workload (where does search time go?)."""
import cProfile, os, pstats, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_eurosys_liumlsmybw24_b200 as A
from aceso_inputs import profiles as P
from paper_conf_eurosys_liumlsmybw24_b200 import search as S
name = sys.argv[1] if len(sys.argv) > 1 else "gpt3-1.3b"
prof = P.WORKLOADS[name]()
ctx = A.Context(prof, 0)
ev = S.GPUEvaluator(ctx)
S.search(prof, ev, budget_s=5, patience=8)  # warm-up (CUDA init, allocations)
pr = cProfile.Profile()
t0 = time.perf_counter()
pr.enable()
res, st = S.search(prof, S.GPUEvaluator(ctx), budget_s=60, patience=8)
pr.disable()
print("search", time.perf_counter() - t0, "s", st["evaluated"], "configs")
pstats.Stats(pr).sort_stats("cumulative").print_stats(18)
