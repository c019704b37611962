#!/bin/bash
# data-on-device DTRSM on 8 logical GPUs: is the bimodal rate a batch-size effect?
mkdir -p gpurun_out
for rep in 1 2 3; do
  for b in 16 4; do
    for n in 16384 32768; do
      XK_BATCH=$b ONLY="dod" REPS=3 ROUTINE=dtrsm N=$n G=8 T=2048 timeout 600 python tools/ablation.py 2>&1 | tail -1 | sed "s/^/batch=$b N=$n | /" >> gpurun_out/dod_batch.txt
    done
  done
done
