#!/bin/bash
# ncu evidence for profiles/: launch list of the bench command + one full capture of a grouped launch
mkdir -p gpurun_out
python -c "from tools.build_native import build_xk; build_xk()"
ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/ncu_launch_bench.json 2>&1
ncu --set full --clock-control none --import-source on -k regex:dgemm_t -s 6 -c 1 -o gpurun_out/prof_batch -f \
    python bench.py --n 16384 --tile 4096 --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full.log 2>&1
tail -1 gpurun_out/ncu_full.log
