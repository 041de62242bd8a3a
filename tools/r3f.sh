run() { env $2 timeout 300 python bench.py --config C5 --rows 800000000 --sub '' --no-e2e --no-cpu --steps 5 > gpurun_out/r3f.json 2>&1; python -c "
import json; d=json.load(open('gpurun_out/r3f.json')); r=d['roofline']; print('$1', round(d['ms_per_step'],2), {k:round(v['avg_launch_ms'],2) for k,v in r['phases'].items() if isinstance(v,dict)})" || tail -3 gpurun_out/r3f.json; }
for i in 1 2; do
run default "X=1"
run minb3 "BLU_GBY_JIT_MINB=3"
run minb4 "BLU_GBY_JIT_MINB=4"
run ctas2 "BLU_GBY_CTAS_PER_SM=2"
run ctas3 "BLU_GBY_CTAS_PER_SM=3"
done
