#!/bin/bash
mkdir -p gpurun_out
./tools/probe_fp64 > gpurun_out/probe_fp64.txt 2>&1
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv -lms 200 > gpurun_out/probe_clocks.csv &
CP=$!
./tools/probe_fp64 >> gpurun_out/probe_fp64.txt 2>&1
kill $CP
python tools/probe_host.py > gpurun_out/probe_host.txt 2>&1
cat gpurun_out/probe_fp64.txt; tail -20 gpurun_out/probe_host.txt
