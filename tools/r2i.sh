O=gpurun_out; mkdir -p $O
for G in 0 48 80 112; do BLU_GBY_L2SHARE=$G timeout 300 python bench.py --config C3 --sub '' --no-e2e --no-cpu --steps 5 > $O/r2i_C3_$G.json 2>&1; python -c "
import json; d=json.load(open('$O/r2i_C3_$G.json')); r=d['roofline']; print('C3 l2share $G', round(d['ms_per_step'],2), {k:round(v['avg_launch_ms'],2) for k,v in r['phases'].items() if isinstance(v,dict)})"; done
BLU_GBY_L2SHARE=80 timeout 600 python -m pytest tests/test_parity_gpu.py -q -x -k "C3 or part" 2>&1 | tail -1
