set -e
for i in 1 2; do
for P in 0 1; do
BLU_GBY_DENSE_PAIR=$P python bench.py --steps 200 --warmup 5 --no-cpu --no-e2e --no-clocks 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('PAIR=$P', round(d['ms_per_step'],4), round(r['avg_launch_ms'],4), round(r['frac'],3), r['kernel'])"
done; done
BLU_GBY_DENSE_PAIR=1 timeout 300 python -m pytest tests/test_parity_gpu.py -q -x -k "config_parity or small_and_ragged" 2>&1 | tail -2
