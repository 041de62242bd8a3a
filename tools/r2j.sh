O=gpurun_out; mkdir -p $O
for c in C3 C3; do timeout 300 python bench.py --config $c --sub '' --no-e2e --no-cpu --steps 5 > $O/r2j_${c}.json 2>&1; python -c "
import json; d=json.load(open('$O/r2j_${c}.json')); r=d['roofline']; print('$c', round(d['ms_per_step'],2), {k:round(v['avg_launch_ms'],2) for k,v in r['phases'].items() if isinstance(v,dict)})"; done
timeout 600 python -m pytest tests/test_parity_gpu.py -q -x -k "C3 or part" 2>&1 | tail -1
