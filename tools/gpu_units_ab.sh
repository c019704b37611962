#!/bin/bash
# A/B: output tiles per CTA (XK_UNITS=1/2) of the unit-stream GEMM kernel vs the one-tile
# kernel of the parent commit (tools/_ab/dgemm_tma_head.cu, extracted before the run)
mkdir -p gpurun_out
K=paper_conf_sc_gautierl21_b200/csrc/kernels/dgemm_tma.cu
cp $K /tmp/dgemm_tma_new.cu
build() { python -c "from tools.build_native import build_xk; build_xk(force=True)" || exit 1; }
for round in 1 2; do
  cp /tmp/dgemm_tma_new.cu $K; XK_NVCC_FLAGS="-DXK_UNITS=2" build
  timeout 900 python tools/gemm_ab.py 2>&1 | tail -1 | sed "s/^/units2 | /" >> gpurun_out/units_ab.txt
  XK_NVCC_FLAGS="-DXK_UNITS=1" build
  timeout 900 python tools/gemm_ab.py 2>&1 | tail -1 | sed "s/^/units1 | /" >> gpurun_out/units_ab.txt
  cp tools/_ab/dgemm_tma_head.cu $K; XK_NVCC_FLAGS="" build
  timeout 900 python tools/gemm_ab.py 2>&1 | tail -1 | sed "s/^/head   | /" >> gpurun_out/units_ab.txt
done
cp /tmp/dgemm_tma_new.cu $K; XK_NVCC_FLAGS="-DXK_UNITS=2" build
timeout 900 python -m pytest tests/test_gpu_kernel.py tests/test_gpu_dgemm.py tests/test_gpu_blas3.py -x -q 2>&1 | tail -2 >> gpurun_out/units_ab.txt
