#!/bin/bash
python -c "from tools.build_native import build_xk; build_xk()"
timeout 600 python -m pytest tests/test_gpu_kernel.py -q -x 2>&1 | tail -1
for g in 0 8 16 32; do XK_GROUP_M=$g python bench.py --n 16384 --tile 4096 --steps 3 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/bg$g.json 2>/dev/null; python -c "
import json; d=json.load(open('gpurun_out/bg$g.json')); print('group_m $g', round(d['value'],2), round(d['roofline']['achieved'],2))"; done
for g in 0 16; do XK_GROUP_M=$g ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct -k regex:dgemm_t -s 6 -c 1 python bench.py --n 16384 --tile 4096 --steps 1 --warmup 1 --no-cpu-baseline --no-e2e 2>&1 | grep -E "dram__bytes|duration|hit_rate" | sed "s/^/g$g /"; done
