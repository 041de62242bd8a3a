"""Phase timing of one config through libblugby (wall clock vs CUDA-event phases). Dev tool."""
import os, sys, time, json
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
if os.environ.get("OLD"):  # same-run A/B: the package built from an earlier revision under _oldpkg/
    sys.path.insert(0, os.path.join(ROOT, "_oldpkg"))
import torch, blugen
from paper_conf_sigmod_merajispcksygnk16_b200 import blugby as bg
cfg = sys.argv[1] if len(sys.argv) > 1 else "C3"
rows = int(sys.argv[2]) if len(sys.argv) > 2 else None
w = blugen.workload(cfg, n_rows=rows) if rows else blugen.workload(cfg)
kc, vc = blugen.device_columns(w)
torch.cuda.synchronize()
plan = bg.plan_for(w.schema, w.est_groups, w.n_rows)
print(json.dumps(plan.info()))
bg.blu_gby_set_timing(True)
flush = torch.empty(512 * 2**20, dtype=torch.uint8, device="cuda") if os.environ.get("FLUSH") else None
for i in range(int(os.environ.get('ITERS', '4'))):
    if flush is not None:
        flush.zero_()
        torch.cuda.synchronize()
    t0 = time.perf_counter()
    r = bg.blu_gby_execute(plan, kc, vc)
    t1 = time.perf_counter()
    t = bg.blu_gby_last_timing()
    print(f"wall {1000*(t1-t0):8.2f} ms  init {t['init_ms']:.2f} agg {t['aggregate_ms']:.2f} compact {t['compact_ms']:.2f} launches {t['aggregate_launches']} retries {t['retries']} groups {r.n_groups}")
    del r
