#!/bin/bash
mkdir -p gpurun_out
python -c "from tools.build_native import build_xk; build_xk()"
ncu --set full --clock-control none --import-source on -k regex:dgemm_tile -s 3 -c 1 -o gpurun_out/prof_tile_${1:-x} -f python tools/tile_bench.py ${2:-4096} 2 > gpurun_out/ncu_full.log 2>&1; tail -2 gpurun_out/ncu_full.log
