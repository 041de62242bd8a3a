timeout 120 python tools/pcie_check.py
BLU_GBY_DEBUG_HOST=1 timeout 300 python -c "
import time, torch, blugen
from paper_conf_sigmod_merajispcksygnk16_b200 import blugby as bg
w = blugen.workload('C5'); m = 250_000_000
kc = [blugen.gen_device(c, w.seed, 0, m, 'cuda') for c in w.key_cols]; vc = [blugen.gen_device(c, w.seed, 0, m, 'cuda') for c in w.val_cols]
hk = [k.cpu().pin_memory() for k in kc]; hv = [v.cpu().pin_memory() for v in vc]
plan = bg.plan_for(w.schema, w.est_groups, m)
r = bg.blu_gby_execute_host(plan, hk, hv); del r
for i in range(3):
    t0 = time.perf_counter(); r = bg.blu_gby_execute_host(plan, hk, hv); t1 = time.perf_counter(); n = r.n_groups; del r; t2 = time.perf_counter()
    print('execute_host %.1f ms, free %.1f ms, groups %d' % ((t1-t0)*1e3, (t2-t1)*1e3, n))
" 2>&1 | tail -8
