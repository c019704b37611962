#!/bin/bash
mkdir -p gpurun_out
python -c "from tools.build_native import build_xk; build_xk()"
python -m pytest tests/test_gpu_kernel.py -q -x 2>&1 | tail -2
for cfg in 0 4 5 6; do
  for T in 2048 4096; do XK_KCFG=$cfg python tools/tile_bench.py $T 10 | sed "s/^/cfg$cfg /"; done
done | tee gpurun_out/kernel_sweep.txt
for tt in "N T" "T N" "T T"; do python tools/tile_bench.py 2048 10 $tt; done | tee -a gpurun_out/kernel_sweep.txt
