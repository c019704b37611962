#!/bin/bash
# A/B of the GEMM epilogue: loads batched per row fragment (EPI_ROWS=1, default), per two
# (EPI_ROWS=2), and the previous interleaved load/store epilogue (tools/_ab/dgemm_tma_old.cu =
# the parent commit's dgemm_tma.cu, extracted before the run)
mkdir -p gpurun_out
K=paper_conf_sc_gautierl21_b200/csrc/kernels/dgemm_tma.cu
cp $K /tmp/dgemm_tma_new.cu
build() { python -c "from tools.build_native import build_xk; build_xk(force=True)" || exit 1; }
for round in 1 2; do
  cp /tmp/dgemm_tma_new.cu $K; XK_NVCC_FLAGS="" build
  timeout 900 python tools/gemm_ab.py 2>&1 | tail -1 | sed "s/^/epi1 | /" >> gpurun_out/epi_ab.txt
  XK_NVCC_FLAGS="-DXK_EPI_ROWS=2" build
  timeout 900 python tools/gemm_ab.py 2>&1 | tail -1 | sed "s/^/epi2 | /" >> gpurun_out/epi_ab.txt
  cp tools/_ab/dgemm_tma_old.cu $K; XK_NVCC_FLAGS="" build
  timeout 900 python tools/gemm_ab.py 2>&1 | tail -1 | sed "s/^/old  | /" >> gpurun_out/epi_ab.txt
done
cp /tmp/dgemm_tma_new.cu $K; XK_NVCC_FLAGS="" build
timeout 900 python -m pytest tests/test_gpu_kernel.py tests/test_gpu_dgemm.py -x -q 2>&1 | tail -2 >> gpurun_out/epi_ab.txt
timeout 900 python tools/bench_blas3.py 2>&1 | tail -1 >> gpurun_out/epi_ab.txt
