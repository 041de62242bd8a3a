# session 4: verify HEAD (JIT constant-offset spec) on the GPU: smoke, GPU tests, every bench line, C2 ncu
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r1h_smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/r1h_smoke.log
python -m pytest tests -m gpu -q > gpurun_out/r1h_gputests.log 2>&1; tail -1 gpurun_out/r1h_gputests.log
python bench.py --steps 200 --warmup 5 > gpurun_out/r1h_bench_C2.json 2> gpurun_out/r1h_bench_C2.err
for c in C1 C3 C4 C5 S1; do
  python bench.py --config $c --steps 10 --warmup 3 > gpurun_out/r1h_bench_$c.json 2> gpurun_out/r1h_bench_$c.err
done
python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/r1h_bench_ref.json 2> gpurun_out/r1h_bench_ref.err
ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/r1h_launches_C2.csv python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:blu_jit_dense -s 3 -c 1 -o gpurun_out/r1h_prof_C2 python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1
ls gpurun_out | grep r1h
