#!/bin/bash
# after the stream-ordered tile allocator: first data-on-device call, GPU suite, bench, DTRSM ablation
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
for n in 16384 32768; do N=$n REPS=4 timeout 600 python tools/dod_reps.py > gpurun_out/dod_reps_after_$n.txt 2>&1; done
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -5 > gpurun_out/gpu_tests.txt
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1 > gpurun_out/smoke.txt
python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
for n in 16384 32768; do
  REPS=3 ROUTINE=dtrsm N=$n G=8 T=2048 timeout 900 python tools/ablation.py > gpurun_out/abl_dtrsm_$n.log 2>&1; tail -1 gpurun_out/abl_dtrsm_$n.log > gpurun_out/ablation_dtrsm_n${n}_g8.json
done
