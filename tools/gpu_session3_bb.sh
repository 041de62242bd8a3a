# shared-table offsets as JIT constants (default) vs kernel parameters (BLU_SOFF_PARAM)
for i in 1 2; do
for D in "NONE" "BLU_SOFF_PARAM"; do
for c in C2 C4; do
BLU_GBY_JIT_DEFS=$D python bench.py --config $c --steps 20 --warmup 3 --no-cpu --no-e2e --no-clocks 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$c $D', round(d['ms_per_step'],4), round(r['avg_launch_ms'],4), round(r['frac'],3))"
done; done; done
python -m pytest tests/test_parity_gpu.py -x -q -k "config_parity or rank_front or forced_paths or small_and_ragged or partitioned" 2>&1 | tail -2
