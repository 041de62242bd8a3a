O=gpurun_out; mkdir -p $O
M="gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct"
for G in 16 4 2 1; do
  BLU_GBY_GRAB=$G timeout 600 ncu --metrics $M --clock-control none -k regex:blu_jit_global_2 -s 3 -c 1 --csv \
    python bench.py --config C5 --rows 400000000 --steps 1 --warmup 3 --no-e2e --no-cpu --sub '' --no-clocks 2>/dev/null | grep -E "gpu__time|dram__|lts__" | awk -F'","' -v p=$G '{print "G="p, $(NF-2), $NF}'
done
for G in 16 2; do BLU_GBY_GRAB=$G timeout 300 python bench.py --config C5 --sub '' --no-e2e --no-cpu --steps 3 > $O/r2h_C5_$G.json 2>&1; python -c "
import json; d=json.load(open('$O/r2h_C5_$G.json')); r=d['roofline']; print('C5 grab $G', round(d['ms_per_step'],2), {k:round(v['avg_launch_ms'],2) for k,v in r['phases'].items() if isinstance(v,dict)})"; done
