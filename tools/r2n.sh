O=gpurun_out; mkdir -p $O
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > $O/r2n_smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/r2n_smoke.log
timeout 1500 python -m pytest tests -m gpu -q -x > $O/r2n_gputests.log 2>&1; echo "tests rc=$?"; tail -2 $O/r2n_gputests.log
timeout 900 python bench.py > $O/r2n_bench.json 2> $O/r2n_bench.err; echo bench rc=$?
