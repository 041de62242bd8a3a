# C4: software-pipelined stream (MODE 3) A/B, with and without the per-warp L2 prefetch
for E in "BLU_GBY_AGG_PREFETCH=1" "BLU_GBY_PIPE=1" "BLU_GBY_PIPE=1 BLU_GBY_AGG_PREFETCH=1" "BLU_GBY_PIPE=1 BLU_GBY_PIPE_R=4" "BLU_GBY_PIPE=1 BLU_GBY_PIPE_R=4 BLU_GBY_AGG_PREFETCH=1"; do
env $E python bench.py --config C4 --steps 10 --warmup 3 --no-cpu --no-e2e --no-clocks 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('C4 $E', round(d['ms_per_step'],3), round(r['avg_launch_ms'],3), round(r['frac'],3), r['kernel'])"
done
for E in "BLU_GBY_X=0" "BLU_GBY_PIPE=1" "BLU_GBY_PIPE=1 BLU_GBY_AGG_PREFETCH=1"; do
env $E python bench.py --config C3 --steps 5 --warmup 2 --no-cpu --no-e2e --no-clocks 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('C3 $E', round(d['ms_per_step'],3), r['kernel'])"
done
BLU_GBY_PIPE=1 BLU_GBY_JIT_VERBOSE=1 python -m pytest tests/test_parity_gpu.py -x -q -k "rank_front or forced_paths or config_parity or small_and_ragged" 2>&1 | tail -2
