#!/bin/bash
# DTRSM / DTRMM host-resident: grouped-launch size and kernel streams (the R10 window turns a
# step's catch-up updates into per-tile chains, so consecutive 16-task batches depend on each
# other; smaller batches let two independent ones overlap)
mkdir -p gpurun_out
for round in 1 2; do
  for cfg in "XK_BATCH=16" "XK_BATCH=8" "XK_BATCH=4" "XK_KSTREAMS=4 XK_BATCH=8"; do
    env $cfg ROUTINES="dtrsm dtrmm" timeout 900 python tools/bench_blas3.py 2>&1 | tail -1 | sed "s/^/$cfg | /" >> gpurun_out/trsm_batch_ab.txt
  done
done
