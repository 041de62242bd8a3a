mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_parity_gpu.py -q -x -k "C3 or part" > gpurun_out/r2g_tests.log 2>&1; tail -1 gpurun_out/r2g_tests.log
timeout 300 python bench.py --config C3 --sub '' --no-e2e --no-cpu --steps 5 > gpurun_out/r2g_bench_C3.json 2>&1
python -c "
import json; d=json.load(open('gpurun_out/r2g_bench_C3.json')); r=d['roofline']; print('C3', round(d['ms_per_step'],2), {k:round(v['avg_launch_ms'],2) for k,v in r['phases'].items() if isinstance(v,dict)})"
for P in 64 256; do
BLU_GBY_PARTS=$P timeout 300 python bench.py --config C5 --sub '' --no-e2e --no-cpu --steps 3 > gpurun_out/r2g_bench_C5_$P.json 2>&1
python -c "
import json; d=json.load(open('gpurun_out/r2g_bench_C5_$P.json')); r=d['roofline']; print('C5 parts $P', round(d['ms_per_step'],2), {k:round(v['avg_launch_ms'],2) for k,v in r['phases'].items() if isinstance(v,dict)})"
done
