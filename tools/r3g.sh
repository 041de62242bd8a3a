run() { env $3 timeout 400 python bench.py --config C5 --rows $2 --sub '' --no-e2e --no-cpu --steps 3 > gpurun_out/r3g.json 2>&1; python -c "
import json; d=json.load(open('gpurun_out/r3g.json')); r=d['roofline']; print('$1 $2', round(d['ms_per_step'],2), {k:round(v['avg_launch_ms'],2) for k,v in r['phases'].items() if isinstance(v,dict)})" || tail -3 gpurun_out/r3g.json; }
for i in 1 2; do
run base 1600000000 "BLU_GBY_OVERLAP=0"
run ovl 1600000000 "BLU_GBY_OVERLAP=1"
done
run base 4000000000 "BLU_GBY_OVERLAP=0"
run ovl 4000000000 "BLU_GBY_OVERLAP=1"
BLU_GBY_OVERLAP=1 BLU_GBY_OVERLAP_MIN=0 timeout 600 python -m pytest tests/test_parity_gpu.py -q -x -k "partition or C5 or C3 or tma_edges" > gpurun_out/r3g_t.log 2>&1; tail -1 gpurun_out/r3g_t.log
