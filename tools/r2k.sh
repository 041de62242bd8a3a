O=gpurun_out; mkdir -p $O
for i in 1 2; do for one in 0 1; do BLU_GBY_2LEVEL_ONE=$one timeout 300 python bench.py --config C3 --sub '' --no-e2e --no-cpu --steps 5 > $O/r2k_C3_$one.json 2>&1; python -c "
import json; d=json.load(open('$O/r2k_C3_$one.json')); r=d['roofline']; print('C3 one=$one', round(d['ms_per_step'],2), {k:round(v['avg_launch_ms'],2) for k,v in r['phases'].items() if isinstance(v,dict)})"; done; done
