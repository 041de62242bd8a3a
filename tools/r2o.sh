O=gpurun_out; mkdir -p $O
for P in 32 16 128; do BLU_GBY_PARTS=$P timeout 300 python bench.py --config C5 --sub '' --no-e2e --no-cpu --steps 3 > $O/r2o_C5_$P.json 2>&1; python -c "
import json; d=json.load(open('$O/r2o_C5_$P.json')); r=d['roofline']; print('C5 parts $P', round(d['ms_per_step'],2), {k:round(v['avg_launch_ms'],2) for k,v in r['phases'].items() if isinstance(v,dict)})"; done
