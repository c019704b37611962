#!/bin/bash
# T=1024 grouped-launch knobs (kernel streams, batch size): data-on-device DGEMM N=32768,
# tools/gemm_ab.py, two alternating rounds
mkdir -p gpurun_out
for round in 1 2; do
  for cfg in "XK_KSTREAMS=2" "XK_KSTREAMS=3" "XK_KSTREAMS=4" "XK_BATCH=8" "XK_KSTREAMS=4 XK_BATCH=8"; do
    env $cfg TILES=1024,2048 timeout 600 python tools/gemm_ab.py 2>&1 | tail -1 | sed "s/^/$cfg | /" >> gpurun_out/t1024_ab.txt
  done
done
# refresh the BLAS-3 table and BASELINE configs[4] on one GPU with the committed defaults
timeout 900 python tools/bench_blas3.py > gpurun_out/blas3.txt 2>&1
timeout 1500 python tools/config5.py > gpurun_out/config5.txt 2>&1
