for c in C3 C5; do timeout 300 python bench.py --config $c --sub '' --no-e2e --no-cpu --steps 3 > gpurun_out/r2r_$c.json 2>&1; python -c "
import json; d=json.load(open('gpurun_out/r2r_$c.json')); r=d['roofline']; print('$c', round(d['ms_per_step'],2), {k:round(v['avg_launch_ms'],2) for k,v in r['phases'].items() if isinstance(v,dict)})"; done
timeout 900 python -m pytest tests/test_parity_gpu.py -q -x -k "C3 or part or fanout or C5" 2>&1 | tail -1
