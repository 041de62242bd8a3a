# session 4 final: smoke, full GPU suite and the default bench line on HEAD
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r1j_smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/r1j_smoke.log
python -m pytest tests -m gpu -q > gpurun_out/r1j_gputests.log 2>&1; tail -1 gpurun_out/r1j_gputests.log
python bench.py > gpurun_out/r1j_bench_C2.json 2> gpurun_out/r1j_bench_C2.err; tail -c 300 gpurun_out/r1j_bench_C2.json
python bench.py --config C4 --steps 10 --warmup 3 > gpurun_out/r1j_bench_C4.json 2> gpurun_out/r1j_bench_C4.err
