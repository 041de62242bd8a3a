"""Per-piece host cost of the Python binding's execute wrapper (dev tool; run on a GPU box)."""
import ctypes, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import blugen
from paper_conf_sigmod_merajispcksygnk16_b200 import blugby as bg

w = blugen.workload("C2", n_rows=1 << 20)
kc, vc = blugen.device_columns(w)
plan = bg.plan_for(w.schema, w.est_groups, w.n_rows)
r = bg.blu_gby_execute(plan, kc, vc)
torch.cuda.synchronize()
N = 2000


def t(name, f):
    for _ in range(50):
        f()
    t0 = time.perf_counter()
    for _ in range(N):
        f()
    print(f"{name:28s} {(time.perf_counter() - t0) / N * 1e6:7.2f} us")


ptr = r.keys[0].data_ptr()
t("current_stream", lambda: torch.cuda.current_stream().cuda_stream)
t("_ptrs x2", lambda: (bg._ptrs(kc), bg._ptrs(vc)))
t("as_tensor(CAI)", lambda: torch.as_tensor(bg._DevArray(None, ptr, 1024, bg.BLU_I64), device="cuda"))
t("as_tensor(CAI, dev obj)", lambda: torch.as_tensor(bg._DevArray(None, ptr, 1024, bg.BLU_I64), device=kc[0].device))
t("_out_dtypes", lambda: bg._out_dtypes(plan, False))
rc = r.c
t("Result(rc) (7 tensors)", lambda: bg.Result.__new__(bg.Result).__init__(rc, bg._key_dtypes(plan), bg._out_dtypes(plan, False), 0, kc[0].device))
t("execute (whole call)", lambda: bg.blu_gby_execute(plan, kc, vc))
