#!/bin/bash
mkdir -p gpurun_out
python -c "from tools.build_native import build_all; build_all()" || exit 1
for r in ${ROUTINES:-dtrsm dtrmm}; do
  for d in 0 1; do
    DOD=$d ROUTINE=$r N=${N:-32768} T=${T:-2048} timeout 300 python tools/trace_routine.py > gpurun_out/trace_${r}_$d.log 2>&1; tail -1 gpurun_out/trace_${r}_$d.log | cut -c1-1500
  done
done
mkdir -p gpurun_out/traces; mv gpurun_out/trace_*_g1*.json gpurun_out/traces/ 2>/dev/null
cd gpurun_out/traces && gzip -f *.json
