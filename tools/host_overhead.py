"""Host-side cost of one small execute (C1): wall time of the C call vs the Python wrapper vs the
device time of the step. Usage: python tools/host_overhead.py [C1|C2] [iters]"""
import ctypes
import sys
import time

import os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import blugen
from paper_conf_sigmod_merajispcksygnk16_b200 import blugby as bg

cfg = sys.argv[1] if len(sys.argv) > 1 else "C1"
iters = int(sys.argv[2]) if len(sys.argv) > 2 else 200
w = blugen.workload(cfg)
kc, vc = blugen.device_columns(w)
plan = bg.plan_for(w.schema, w.est_groups, w.n_rows)
s = torch.cuda.current_stream()
for _ in range(10):
    bg.blu_gby_execute(plan, kc, vc, stream=s)
torch.cuda.synchronize()
kp, vp = bg._ptrs(kc), bg._ptrs(vc)
sh = bg._stream_handle(s)
t0 = time.perf_counter()
for _ in range(iters):
    rc = bg.ResultC()
    bg.lib.blu_gby_execute(plan.handle, kp, vp, w.n_rows, sh, ctypes.byref(rc))
    bg.lib.blu_gby_result_free(ctypes.byref(rc), sh)
torch.cuda.synchronize()
c_us = (time.perf_counter() - t0) / iters * 1e6
t0 = time.perf_counter()
for _ in range(iters):
    r = bg.blu_gby_execute(plan, kc, vc, stream=s)
    del r
torch.cuda.synchronize()
py_us = (time.perf_counter() - t0) / iters * 1e6
bg.blu_gby_set_timing(True)
bg.blu_gby_execute(plan, kc, vc, stream=s)
t = bg.blu_gby_last_timing()
print({"config": cfg, "c_call_us": round(c_us, 1), "python_call_us": round(py_us, 1),
       "device_total_us": round(t["total_ms"] * 1e3, 1), "aggregate_us": round(t["aggregate_ms"] * 1e3, 1),
       "kernel": t["kernel"]})
