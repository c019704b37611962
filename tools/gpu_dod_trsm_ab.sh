#!/bin/bash
# data-on-device DTRSM N=32768 on 8 logical GPUs: planner window and task rate (what made
# round-2's DoD row drop against round 1's)
mkdir -p gpurun_out
python -c "from tools.build_native import build_all; build_all()" || exit 1
for cfg in "XK_WINDOW=4" "XK_WINDOW=2" "XK_WINDOW=4 XK_TASK_RATE=29000000" "XK_WINDOW=2 XK_TASK_RATE=29000000"; do
  env $cfg ONLY="full dod" ROUTINE=dtrsm N=32768 G=8 T=2048 timeout 900 python tools/ablation.py 2>&1 | tail -1 | sed "s/^/$cfg | /" >> gpurun_out/dod_trsm_ab.txt
done
for cfg in "XK_WINDOW=4" "XK_WINDOW=2"; do
  env $cfg ONLY="full dod" ROUTINE=dgemm N=32768 G=8 T=2048 timeout 900 python tools/ablation.py 2>&1 | tail -1 | sed "s/^/$cfg dgemm | /" >> gpurun_out/dod_trsm_ab.txt
done
# the per-call batch cap (R19) with the committed defaults
ROUTINES="dtrsm dtrmm dgemm" timeout 900 python tools/bench_blas3.py 2>&1 | tail -1 | sed "s/^/R19 | /" >> gpurun_out/dod_trsm_ab.txt
ROUTINES="dtrsm dtrmm" timeout 900 python tools/bench_blas3.py 2>&1 | tail -1 | sed "s/^/R19 | /" >> gpurun_out/dod_trsm_ab.txt
timeout 1200 python -m pytest tests/test_gpu_blas3.py tests/test_gpu_rank.py tests/test_gpu_fuzz.py -x -q 2>&1 | tail -2 >> gpurun_out/dod_trsm_ab.txt
