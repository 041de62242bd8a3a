timeout 900 python -m pytest tests/test_parity_gpu.py -q -x -k "minmax_skip or rank_front or small_and_ragged or config_parity or hot_reg or forced_paths" > gpurun_out/r4d_t.log 2>&1; echo tests rc=$?; tail -2 gpurun_out/r4d_t.log
bash tools/ab_cfg.sh C4 BLU_GBY_MMBOUND=0 BLU_GBY_MMBOUND=1
bash tools/ab_cfg.sh C2 BLU_GBY_MMBOUND=0 BLU_GBY_MMBOUND=1
