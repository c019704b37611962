#!/bin/bash
mkdir -p gpurun_out
python -c "from tools.build_native import build_xk; build_xk()"
ncu --set full --clock-control none --import-source on -k regex:dgemm_t -s 6 -c 1 -o gpurun_out/prof_batch -f \
    python bench.py --n 16384 --tile 4096 --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full.log 2>&1
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed,sm__throughput.avg.pct_of_peak_sustained_elapsed \
    -k regex:trxm_base --csv --log-file gpurun_out/trsm_base.csv python tools/trsm_panel.py > /dev/null 2>&1
ncu --metrics gpu__time_duration.sum --csv --log-file gpurun_out/trsm_launches.csv python tools/trsm_panel.py > /dev/null 2>&1
echo done
