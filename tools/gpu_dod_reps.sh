#!/bin/bash
mkdir -p gpurun_out
for n in 16384 32768; do N=$n REPS=8 timeout 600 python tools/dod_reps.py > gpurun_out/dod_reps_$n.txt 2>&1; done
N=16384 REPS=8 XK_KSTREAMS=1 timeout 600 python tools/dod_reps.py > gpurun_out/dod_reps_16384_ks1.txt 2>&1
