# C3: pipelined pass 2 (MODE 4) and pipelined scatter A/B
for E in "BLU_GBY_X=0" "BLU_GBY_SEG_PIPE=1" "BLU_GBY_SCATTER_PIPE=1" "BLU_GBY_SCATTER_PIPE=1 BLU_GBY_PREFETCH=0" "BLU_GBY_SEG_PIPE=1 BLU_GBY_SCATTER_PIPE=1"; do
env $E python bench.py --config C3 --steps 5 --warmup 2 --no-cpu --no-e2e --no-clocks 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('C3 $E', round(d['ms_per_step'],3), r.get('phases'))"
done
BLU_GBY_SEG_PIPE=1 BLU_GBY_SCATTER_PIPE=1 python -m pytest tests/test_parity_gpu.py -x -q -k "C3 or C5 or partition or est_groups or regrow" 2>&1 | tail -2
