"""cProfile of the Python execute wrapper on C2 (dev tool; run on a GPU box)."""
import cProfile, os, pstats, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import blugen
from paper_conf_sigmod_merajispcksygnk16_b200 import blugby as bg

w = blugen.workload("C2")
kc, vc = blugen.device_columns(w)
plan = bg.plan_for(w.schema, w.est_groups, w.n_rows)
s = torch.cuda.current_stream()
for _ in range(5):
    r = bg.blu_gby_execute(plan, kc, vc, stream=s)
    del r
torch.cuda.synchronize()
pr = cProfile.Profile()
pr.enable()
t0 = time.perf_counter()
for _ in range(50):
    r = bg.blu_gby_execute(plan, kc, vc, stream=s)
    del r
torch.cuda.synchronize()
pr.disable()
print("per call us", (time.perf_counter() - t0) / 50 * 1e6)
pstats.Stats(pr).sort_stats("tottime").print_stats(12)
