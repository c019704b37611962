#!/bin/bash
# paper Table II on 8 logical GPUs (one B200): DGEMM / DSYR2K / DTRSM, every heuristic mode + DoD
mkdir -p gpurun_out
python -c "from tools.build_native import build_all; build_all()" || exit 1
for r in ${ROUTINES:-dgemm dsyr2k dtrsm}; do
  for n in ${NS:-16384 32768}; do
    ROUTINE=$r N=$n G=8 T=2048 timeout 900 python tools/ablation.py > gpurun_out/abl_${r}_$n.log 2>&1; tail -1 gpurun_out/abl_${r}_$n.log > gpurun_out/ablation_${r}_n${n}_g8.json; cat gpurun_out/ablation_${r}_n${n}_g8.json | cut -c1-300; python -c "import json;print(json.load(open('gpurun_out/ablation_${r}_n${n}_g8.json'))['vs_full_percent'])"
  done
done
