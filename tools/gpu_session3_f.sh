# dense path (a) pipelined stream A/B (C2, C1); one-pass hash path (K3) with MODE 3
for i in 1 2; do
for E in "BLU_GBY_X=0" "BLU_GBY_DENSE_PIPE=1" "BLU_GBY_DENSE_PIPE=1 BLU_GBY_DENSE_PIPE_R=4"; do
env $E python bench.py --config C2 --steps 30 --warmup 3 --no-cpu --no-e2e --no-clocks 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('C2 $E', round(d['ms_per_step'],4), round(r['avg_launch_ms'],4), round(r['frac'],3), r['kernel'])"
done; done
for E in "BLU_GBY_X=0" "BLU_GBY_DENSE_PIPE=1"; do
env $E python bench.py --config C1 --steps 30 --warmup 3 --no-cpu --no-e2e --no-clocks 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('C1 $E', round(d['ms_per_step'],4), round(r['avg_launch_ms'],4), round(r['frac'],3), r['kernel'])"
done
for E in "BLU_GBY_X=0" "BLU_GBY_PIPE=1"; do
env $E ITERS=4 python tools/phase_probe.py K3 2>&1 | tail -2 | sed "s/^/K3 $E /"
done
BLU_GBY_DENSE_PIPE=1 BLU_GBY_PIPE=1 python -m pytest tests/test_parity_gpu.py -x -q 2>&1 | tail -2
