"""Device time of the S10 owner partition (blu_gby_partition on a C5-shaped partial, and
blu_gby_partition_rows on C3-shaped rows) for P owners. Usage: python tools/partition_probe.py [old]
("old" imports the package from _oldpkg/, a build of an earlier revision, for same-run A/B)."""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if len(sys.argv) > 1 and sys.argv[1] == "old":
    sys.path.insert(0, os.path.join(ROOT, "_oldpkg"))
sys.path.insert(1, ROOT)
import torch

import blugen
from paper_conf_sigmod_merajispcksygnk16_b200 import blugby as bg

tag = sys.argv[1] if len(sys.argv) > 1 else "new"
s = torch.cuda.current_stream()


def timed(f, iters=5):
    f()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t0 = time.perf_counter()
    e0.record(s)
    for _ in range(iters):
        f()
    e1.record(s)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / iters, (time.perf_counter() - t0) / iters * 1e3


w = blugen.workload("C5", n_rows=400_000_000, n_groups=50_000_000)
kc, vc = blugen.device_columns(w)
plan = bg.plan_for(w.schema, w.est_groups, w.n_rows)
part = bg.blu_gby_execute_partial(plan, kc, vc, stream=s)
del kc, vc
words = plan.record_bytes // 8
for P in (2, 8):
    send = torch.empty(part.n_groups * words, dtype=torch.int64, device="cuda")
    dev_ms, wall_ms = timed(lambda: bg.blu_gby_partition(plan, part, P, send, stream=s))
    print(f"{tag} partition partial C5 {part.n_groups} records P={P}: {dev_ms:.3f} ms (wall {wall_ms:.3f})")
    del send
del part
w = blugen.workload("C3", n_rows=100_000_000)
kc, vc = blugen.device_columns(w)
plan = bg.plan_for(w.schema, w.est_groups, w.n_rows)
words = plan.row_record_bytes // 8
send = torch.empty(w.n_rows * words, dtype=torch.int64, device="cuda")
for P in (2, 8):
    dev_ms, wall_ms = timed(lambda: bg.blu_gby_partition_rows(plan, kc, vc, P, send, stream=s))
    print(f"{tag} partition rows C3 {w.n_rows} rows P={P}: {dev_ms:.3f} ms (wall {wall_ms:.3f})")
