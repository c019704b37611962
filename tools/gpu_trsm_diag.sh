#!/bin/bash
# TRSM/TRMM investigation: host-resident timelines + ncu of the diagonal-tile base kernel
mkdir -p gpurun_out
python -c "from tools.build_native import build_all; build_all()" || exit 1
for r in dtrsm dtrmm dgemm; do
  ROUTINE=$r N=32768 T=2048 timeout 300 python tools/trace_routine.py > gpurun_out/trace_$r.log 2>&1; tail -1 gpurun_out/trace_$r.log
done
rm -f gpurun_out/trace_*_g1.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/trsm_launches.csv python tools/trsm_panel.py > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:trxm_base -s 3 -c 1 -f -o gpurun_out/trsm_base python tools/trsm_panel.py > /dev/null 2>&1
ls -la gpurun_out
