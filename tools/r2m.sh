timeout 120 python tools/host_overhead.py C1 500 2>&1 | tail -1
for c in 2 1; do BLU_GBY_CTAS_PER_SM=$c timeout 300 python bench.py --config C1 --sub '' --no-e2e --no-cpu --steps 300 > gpurun_out/r2m_C1_$c.json 2>&1; python -c "
import json; d=json.load(open('gpurun_out/r2m_C1_$c.json')); r=d['roofline']; print('C1 ctas $c', round(d['ms_per_step'],4), round(r['avg_launch_ms'],4))"; done
timeout 600 python -m pytest tests/test_parity_gpu.py -q -x -k "C1 or C2 or host" 2>&1 | tail -1
