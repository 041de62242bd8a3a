O=gpurun_out; mkdir -p $O
timeout 120 python tools/host_overhead.py C1 500
BLU_GBY_DEBUG_HOST=1 timeout 120 python tools/host_overhead.py C1 3 2>&1 | tail -12
timeout 300 python bench.py --config C3 --sub '' --no-e2e --no-cpu --steps 5 > $O/r2m_C3.json 2>&1; python -c "
import json; d=json.load(open('$O/r2m_C3.json')); r=d['roofline']; print('C3', round(d['ms_per_step'],2), {k:round(v['avg_launch_ms'],2) for k,v in r['phases'].items() if isinstance(v,dict)})"
timeout 300 python bench.py --config C1 --sub '' --no-e2e --no-cpu --steps 200 > $O/r2m_C1.json 2>&1; python -c "
import json; d=json.load(open('$O/r2m_C1.json')); r=d['roofline']; print('C1', round(d['ms_per_step'],4), round(r['avg_launch_ms'],4))"
