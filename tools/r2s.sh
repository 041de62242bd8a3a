export BLU_GBY_JIT_VERBOSE=1
for t in 0 1; do for c in C3 C5; do BLU_GBY_SCATTER_TMA=$t timeout 300 python bench.py --config $c --sub '' --no-e2e --no-cpu --steps 3 > gpurun_out/r2s_${c}_$t.json 2>gpurun_out/r2s_${c}_$t.err; python -c "
import json; d=json.load(open('gpurun_out/r2s_${c}_$t.json')); r=d['roofline']; print('$c tma $t', round(d['ms_per_step'],2), {k:round(v['avg_launch_ms'],2) for k,v in r['phases'].items() if isinstance(v,dict)}, d['config']['groups'])" || tail -3 gpurun_out/r2s_${c}_$t.err; done; done
BLU_GBY_SCATTER_TMA=1 timeout 900 python -m pytest tests/test_parity_gpu.py -q -x -k "C3 or part or fanout or C5" 2>&1 | tail -2
