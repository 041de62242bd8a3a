# session 4: two hot keys with compile-time key indices (partials kept in registers) — A/B on C4
mkdir -p gpurun_out
O=gpurun_out/r1i_hotreg2b.txt
: > $O
BLU_GBY_HOT_REG=2 python -m pytest tests/test_parity_gpu.py -q -k "hot_reg or rank_front or forced_paths or config_parity" 2>&1 | tail -1 >> $O
for rep in 1 2; do
for cfg in "1 640" "2 640" "2 576" "2 512"; do
  set -- $cfg
  echo "== HOT_REG=$1 BLOCK=$2 rep=$rep" >> $O
  BLU_GBY_HOT_REG=$1 BLU_GBY_BLOCK=$2 python bench.py --config C4 --steps 10 --warmup 3 --no-e2e --no-cpu 2>>$O | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); r=d['roofline']; print(d['ms_per_step'], r['avg_launch_ms'], r['kernel'], d['config']['block'], r['frac'])" >> $O 2>&1
done
done
cat $O
