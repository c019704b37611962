#!/bin/bash
# full GPU pass + BLAS-3 table refresh
./tools/gpu_round.sh "$@"
timeout 1200 python tools/bench_blas3.py > gpurun_out/blas3.json 2> gpurun_out/blas3.err; tail -1 gpurun_out/blas3.json
