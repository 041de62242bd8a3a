"""Small cases of every path for compute-sanitizer (memcheck / racecheck / synccheck). Dev tool."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, blugen
from paper_conf_sigmod_merajispcksygnk16_b200 import blugby as bg
cases = [("C1", dict(n_rows=100_003), None), ("C2", dict(n_rows=200_011), None), ("C2", dict(n_rows=100_000), "b"),
         ("C3", dict(n_rows=300_003, n_groups=20_000), None), ("C4", dict(n_rows=300_017), None),
         ("C3", dict(n_rows=300_003, n_groups=20_000), "parts")]
for name, kw, mode in cases:
    env = {}
    if mode == "b": os.environ["BLU_GBY_FORCE_PATH"] = "b"
    if mode == "parts": os.environ["BLU_GBY_PARTS"] = "8"
    w = blugen.workload(name, **kw)
    kc, vc = blugen.device_columns(w)
    plan = bg.plan_for(w.schema, w.est_groups, w.n_rows)
    r = bg.blu_gby_execute(plan, kc, vc)
    p = bg.blu_gby_execute_partial(plan, kc, vc)
    m = bg.blu_gby_merge(plan, [p, p])
    torch.cuda.synchronize()
    print(name, mode, plan.info()["path_name"], r.n_groups, m.n_groups, flush=True)
    os.environ.pop("BLU_GBY_FORCE_PATH", None); os.environ.pop("BLU_GBY_PARTS", None)
est, ex = bg.blu_gby_estimate_groups(w.schema.keys, kc, k=256)
print("kmv", est, ex)
