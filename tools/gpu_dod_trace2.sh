#!/bin/bash
# catch a slow data-on-device DTRSM on 8 logical GPUs in the library trace (ablation's sequence)
mkdir -p gpurun_out
for i in 1 2 3 4 5; do
  SYNC_WARMUP=1 XK_BATCH=4 ROUTINE=dtrsm N=16384 G=8 DOD=1 OUT=gpurun_out/slow$i timeout 600 python tools/trace_routine.py > gpurun_out/slow$i.log 2>&1
  tail -1 gpurun_out/slow$i.log | cut -c1-200
done
