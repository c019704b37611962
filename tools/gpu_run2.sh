#!/bin/bash
mkdir -p gpurun_out
timeout 900 python tools/model_fidelity.py > gpurun_out/fidelity.jsonl 2> gpurun_out/fidelity.err
for dod in 0 1; do ROUTINE=dtrsm DOD=$dod timeout 300 python tools/trace_routine.py > gpurun_out/trace_dtrsm_$dod.log 2>&1; done
ROUTINE=dgemm T=2048 timeout 300 python tools/trace_routine.py > gpurun_out/trace_dgemm_0.log 2>&1
GMS="16 32 64" bash tools/gpu_groupm.sh
rm -f gpurun_out/trace_*_n32768_g1*.json.bak
