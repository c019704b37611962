#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
for n in 16384 32768; do
  REPS=5 ROUTINE=dtrsm N=$n G=8 T=2048 timeout 900 python tools/ablation.py > gpurun_out/abl_dtrsm_$n.log 2>&1; tail -1 gpurun_out/abl_dtrsm_$n.log > gpurun_out/ablation_dtrsm_n${n}_g8.json
done
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -3 > gpurun_out/gpu_tests.txt
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1 > gpurun_out/smoke.txt
