mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
for c in C5 C3 C4; do
  timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/r2a_bench_$c.json 2> gpurun_out/r2a_bench_$c.err
  echo "$c rc=$?"; tail -c 400 gpurun_out/r2a_bench_$c.json; echo
done
nproc; grep -m1 "model name" /proc/cpuinfo
