timeout 600 python -m pytest tests/test_parity_gpu.py -q -x -k "rank_front" 2>&1 | tail -1
for i in 1 2; do for d in 0 1; do BLU_GBY_DEDUPE=$d timeout 300 python bench.py --config C4 --sub '' --no-e2e --no-cpu --steps 10 > gpurun_out/r2p_C4_$d.json 2>&1; python -c "
import json; d=json.load(open('gpurun_out/r2p_C4_$d.json')); r=d['roofline']; print('C4 dedupe $d', round(d['ms_per_step'],3), round(r['avg_launch_ms'],3), round(r['frac'],3))"; done; done
