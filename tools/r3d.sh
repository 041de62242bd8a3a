for i in 1 2; do for r in 4 2; do BLU_GBY_BUCKET_R=$r timeout 300 python bench.py --config C3 --sub '' --no-e2e --no-cpu --steps 5 > gpurun_out/r3d.json 2>&1; python -c "
import json; d=json.load(open('gpurun_out/r3d.json')); r=d['roofline']; print('C3 R=$r', round(d['ms_per_step'],2), {k:round(v['avg_launch_ms'],2) for k,v in r['phases'].items() if isinstance(v,dict)})"; done; done
