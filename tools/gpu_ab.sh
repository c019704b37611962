#!/bin/bash
mkdir -p gpurun_out
python -c "from tools.build_native import build_xk; build_xk()"
python -m pytest tests/test_gpu_kernel.py -q -x 2>&1 | tail -1
for rep in 1 2; do for cfg in 4 5 6; do XK_KCFG=$cfg python tools/tile_bench.py 4096 30 | sed "s/^/cfg$cfg /"; done; done | tee gpurun_out/kernel_ab.txt
for ks in 1 2; do XK_KCFG=${CFG:-4} python bench.py --steps 3 --warmup 2 --no-e2e --no-cpu-baseline --kstreams $ks > gpurun_out/bench_ks$ks.json 2>/dev/null; python -c "
import json; d=json.load(open('gpurun_out/bench_ks$ks.json')); print('kstreams $ks value', round(d['value'],2), 'roof', round(d['roofline']['achieved'],2), d['roofline']['per_launch'][-40:])"; done
