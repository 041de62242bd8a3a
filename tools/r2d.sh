mkdir -p gpurun_out
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2d_smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/r2d_smoke.log
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/r2d_gputests.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/r2d_gputests.log
