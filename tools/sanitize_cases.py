"""Small cases of every path for compute-sanitizer (memcheck / racecheck / synccheck). Dev tool."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, blugen
from paper_conf_sigmod_merajispcksygnk16_b200 import blugby as bg
cases = [("C1", dict(n_rows=100_003), None), ("C2", dict(n_rows=200_011), None), ("C2", dict(n_rows=100_000), "b"),
         ("C3", dict(n_rows=300_003, n_groups=20_000), None), ("C4", dict(n_rows=300_017), None),
         ("C3", dict(n_rows=300_003, n_groups=20_000), "parts"),
         ("C3", dict(n_rows=300_003, n_groups=20_000), "parts_smem"),
         ("C4", dict(n_rows=300_017), "front"),
         ("C3", dict(n_rows=1_000_003, n_groups=300_000), "parts_smem")]
for name, kw, mode in cases:
    env = {}
    if mode == "b": os.environ["BLU_GBY_FORCE_PATH"] = "b"
    if mode in ("parts", "parts_smem"): os.environ["BLU_GBY_PARTS"] = "8"
    if mode == "parts_smem": os.environ["BLU_GBY_PART_SMEM"] = "1"
    if mode == "front": os.environ["BLU_GBY_FORCE_PATH"], os.environ["BLU_GBY_HOT_FRONT"] = "d", "1"
    w = blugen.workload(name, **kw)
    kc, vc = blugen.device_columns(w)
    plan = bg.plan_for(w.schema, w.est_groups, w.n_rows)
    r = bg.blu_gby_execute(plan, kc, vc)
    p = bg.blu_gby_execute_partial(plan, kc, vc)
    m = bg.blu_gby_merge(plan, [p, p])
    torch.cuda.synchronize()
    inf = plan.info()
    print(name, mode, inf["path_name"], inf.get("hot_front"), inf.get("parts"), inf.get("bucket_S"), r.n_groups, m.n_groups, flush=True)
    os.environ.pop("BLU_GBY_FORCE_PATH", None); os.environ.pop("BLU_GBY_PARTS", None); os.environ.pop("BLU_GBY_PART_SMEM", None)
    os.environ.pop("BLU_GBY_HOT_FRONT", None)
est, ex = bg.blu_gby_estimate_groups(w.schema.keys, kc, k=256)
print("kmv", est, ex)

# rows-mode exchange (4 simulated owners)
w = blugen.workload("C3", n_rows=200_003, n_groups=20_000)
kc, vc = blugen.device_columns(w)
plan = bg.plan_for(w.schema, w.est_groups, w.n_rows)
buf = torch.empty(w.n_rows * plan.row_record_bytes // 8, dtype=torch.int64, device="cuda")
counts = bg.blu_gby_partition_rows(plan, kc, vc, 4, buf)
r = bg.blu_gby_execute_records(plan, buf, sum(counts))
torch.cuda.synchronize()
print("rows mode", counts, r.n_groups, flush=True)
# 128-bit payloads
rng = np.random.default_rng(1)
n = 100_003
k = rng.integers(0, 2**40, 3000, dtype=np.int64)[rng.integers(0, 3000, n)]
v = np.ascontiguousarray(np.stack([rng.integers(-(2**63), 2**63, n, dtype=np.int64)] * 2, axis=1))
sch = blugen.Schema([(blugen.I64, 0)], [blugen.I128], [(blugen.COUNT, -1), (blugen.SUM, 0), (blugen.MIN, 0),
                                                         (blugen.MAX, 0), (blugen.AVG, 0)])
pq = bg.plan_for(sch, 3000, n)
dk, dv = [torch.from_numpy(k).cuda()], [torch.from_numpy(v).cuda()]
r = bg.blu_gby_execute(pq, dk, dv)
m = bg.blu_gby_merge(pq, [bg.blu_gby_execute_partial(pq, dk, dv)] * 2)
torch.cuda.synchronize()
print("i128", r.n_groups, m.n_groups, flush=True)
# sort offload
rows = blugen.sort_rows(300_007, 16)
perm, st = bg.blu_sort_rows(torch.from_numpy(rows).cuda())
ko, po = bg.blu_sort_pairs(bg.blu_sort_partial_keys(torch.from_numpy(rows).cuda(), 0),
                           torch.arange(300_007, dtype=torch.int32, device="cuda"))
rs, rl = bg.blu_sort_dup_ranges(ko)
torch.cuda.synchronize()
print("sort", st["levels"], st["active"], int(rs.numel()), flush=True)
