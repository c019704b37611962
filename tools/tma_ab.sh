#!/bin/bash
mkdir -p gpurun_out
python -c "from tools.build_native import build_xk; build_xk()"
timeout 600 python -m pytest tests/test_gpu_kernel.py -q -x 2>&1 | tail -1
for T in 2048 4096; do python tools/tile_bench.py $T 20; done
for tt in "N T" "T N" "T T"; do python tools/tile_bench.py 4096 10 $tt; done
ncu --set full --clock-control none -k regex:dgemm_tma -s 3 -c 1 -o gpurun_out/prof_tma -f python tools/tile_bench.py 4096 3 > /dev/null 2>&1; echo ncu done
