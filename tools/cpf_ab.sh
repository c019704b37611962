#!/bin/bash
# A/B: epilogue C prefetch lead (XK_CPF k-blocks before the last two; 1000000 = off)
mkdir -p gpurun_out
for V in 1000000 0 6 1000000 0 6; do
  touch paper_conf_sc_gautierl21_b200/csrc/kernels/dgemm_tma.cu
  NVCC_APPEND_FLAGS="-DXK_CPF=$V" python -c "from tools.build_native import build_xk; build_xk()" || exit 1
  echo "CPF=$V $(python tools/tile_bench.py 4096 20 2>/dev/null | tail -1)"
  timeout 600 python bench.py --steps 3 --warmup 2 --no-cpu-baseline --no-e2e 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('CPF=$V value %.3f kernel frac %.4f' % (d['value'], d['roofline']['frac']))"
done
