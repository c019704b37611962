#!/bin/bash
mkdir -p gpurun_out
python -m pytest tests/test_gpu_kernel.py -m gpu -x -q -s 2>&1 | tail -30 | tee gpurun_out/gpu_kernel_test.txt
