#!/bin/bash
# data-on-device DTRSM N=32768 on 8 logical GPUs: repeated traced calls (what differs between
# a fast and a slow run), then the DTRSM rows of the ablation with the final code
mkdir -p gpurun_out
python -c "from tools.build_native import build_all; build_all()" || exit 1
for i in 1 2 3 4; do
  ROUTINE=dtrsm N=32768 G=8 DOD=1 OUT=gpurun_out/dodtrace$i timeout 600 python tools/trace_routine.py > gpurun_out/dodtrace$i.log 2>&1
  rm -f gpurun_out/dodtrace$i/trace_dtrsm_n32768_g8_dod.json.gz
done
for n in 16384 32768; do
  REPS=5 ROUTINE=dtrsm N=$n G=8 T=2048 timeout 900 python tools/ablation.py > gpurun_out/abl_dtrsm_$n.log 2>&1; tail -1 gpurun_out/abl_dtrsm_$n.log > gpurun_out/ablation_dtrsm_n${n}_g8.json
done
