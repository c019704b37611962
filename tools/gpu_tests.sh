#!/bin/bash
# usage: tools/gpu_tests.sh [pytest args]
mkdir -p gpurun_out
python -c "from tools.build_native import build_all; build_all()"
timeout 1500 python -m pytest tests -m gpu -x -q -s "$@" 2>&1 | tail -40 | tee gpurun_out/gpu_tests.txt
