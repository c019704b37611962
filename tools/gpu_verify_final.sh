#!/bin/bash
# parity of the single-buffered-B GEMM first; the full verification + evidence on the variant
# that passes (XK_FB1=1 if green, else the double-buffered XK_FB1=0)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 1200 python -m pytest tests/test_gpu_kernel.py tests/test_gpu_dgemm.py tests/test_gpu_blas3.py tests/test_gpu_fuzz.py -x -q 2>&1 | tail -3 > gpurun_out/fb1_parity.txt
python -c "import __graft_entry__ as g; g.smoke()" >> gpurun_out/fb1_parity.txt 2>&1
if grep -q "passed" gpurun_out/fb1_parity.txt && ! grep -q "failed\|Error" gpurun_out/fb1_parity.txt; then
  echo "variant FB1=1" > gpurun_out/variant.txt
else
  echo "variant FB1=0 (FB1=1 failed parity)" > gpurun_out/variant.txt
  XK_NVCC_FLAGS="-DXK_FB1=0" python -c "from tools.build_native import build_xk; build_xk(force=True)" || exit 1
fi
bash tools/gpu_final.sh
