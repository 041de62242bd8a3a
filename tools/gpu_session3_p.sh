# warp-per-range sort + unrolled level-key gathers (S1) vs window-only and radix-only
timeout 600 python -m pytest tests/test_sort_gpu.py -x -q 2>&1 | tail -2
for E in "BLU_SORT_X=0" "BLU_SORT_NO_WARP=1" "BLU_SORT_NO_SEG=1"; do
env $E python bench.py --config S1 --steps 5 --warmup 3 --no-cpu --no-e2e --no-clocks 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('S1 $E', round(d['ms_per_step'],3), round(r['avg_launch_ms'],4), [round(x,2) for x in r['ms_per_level'][:4]], r['launches_per_step'])"
done
