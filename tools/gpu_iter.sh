#!/bin/bash
# iteration pass: build, a subset of GPU tests (PYTEST_K), traces, blas3 throughput
mkdir -p gpurun_out
python -c "from tools.build_native import build_all; build_all()" || exit 1
if [ -n "$PYTEST_K" ]; then timeout 900 python -m pytest tests -m gpu -x -q -k "$PYTEST_K" 2>&1 | tail -5 | tee gpurun_out/gpu_tests_iter.txt; fi
if [ -n "$ROUTINES" ]; then bash tools/gpu_trace2.sh; fi
if [ -n "$BLAS3" ]; then timeout 900 python tools/bench_blas3.py 2>&1 | tail -1 | tee gpurun_out/blas3.json; fi
