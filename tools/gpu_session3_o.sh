# window sizes of the segmented window sort vs the batched radix sort (S1)
timeout 600 python -m pytest tests/test_sort_gpu.py -x -q 2>&1 | tail -2
for E in "BLU_SORT_SEG_W=2048" "BLU_SORT_SEG_W=4096" "BLU_SORT_NO_SEG=1"; do
env $E python bench.py --config S1 --steps 5 --warmup 3 --no-cpu --no-e2e --no-clocks 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('S1 $E', round(d['ms_per_step'],3), round(r['avg_launch_ms'],4), r['ms_per_level'], r['launches_per_step'])"
done
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_seg_window|k_rs_downsweep|k_level|k_dup|k_seg" --csv --log-file gpurun_out/s3o_launches_S1.csv python bench.py --config S1 --steps 1 --warmup 1 --no-cpu --no-e2e --no-clocks > /dev/null 2>&1
