#!/bin/bash
mkdir -p gpurun_out
for pool in 1 0; do
  for n in 16384 32768; do XK_POOL=$pool N=$n REPS=3 timeout 600 python tools/dod_reps.py 2>&1 | grep rep | sed "s/^/pool=$pool N=$n | /" >> gpurun_out/dod_reps2.txt; done
done
