#!/bin/bash
# DTRSM / DTRMM host-resident with the untouched dimension processed in column groups (A/B)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
for round in 1 2; do
  for cg in 0 2 4; do
    XK_TRXM_CG=$cg ROUTINES="dtrsm dtrmm" timeout 900 python tools/bench_blas3.py 2>&1 | tail -1 | sed "s/^/cg=$cg | /" >> gpurun_out/trxm_cg.txt
  done
done
XK_TRXM_CG=2 timeout 900 python -m pytest tests/test_gpu_blas3.py -x -q 2>&1 | tail -2 >> gpurun_out/trxm_cg.txt
