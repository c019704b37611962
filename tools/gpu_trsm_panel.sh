#!/bin/bash
# TRSM diagonal-tile ("panel") evidence: launch list + one full ncu capture of the base kernel
mkdir -p gpurun_out
python -c "from tools.build_native import build_all; build_all()" || exit 1
if [ -n "$PYTEST_K" ]; then timeout 900 python -m pytest tests -m gpu -x -q -k "$PYTEST_K" 2>&1 | tail -5 | tee gpurun_out/gpu_tests_iter.txt; fi
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/trsm_launches.csv python tools/trsm_panel.py > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:trxm_base -s 3 -c 1 -f -o gpurun_out/trsm_base python tools/trsm_panel.py > /dev/null 2>&1
