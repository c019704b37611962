#!/bin/bash
# smoke + bench + ncu launch list + ncu full capture of the tile kernel
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.txt 2>&1; tail -2 gpurun_out/smoke.txt
for T in 2048 4096; do python tools/tile_bench.py $T 10; done | tee gpurun_out/tile_bench.txt
python bench.py "$@" > gpurun_out/bench.json 2> gpurun_out/bench.err; tail -3 gpurun_out/bench.err; cat gpurun_out/bench.json
ncu --set full --clock-control none --import-source on -k regex:dgemm_tile -s 3 -c 1 -o gpurun_out/prof_tile -f python tools/tile_bench.py 2048 2 > gpurun_out/ncu_full.log 2>&1; tail -2 gpurun_out/ncu_full.log
ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file gpurun_out/launches.csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/ncu_launch_bench.json 2>&1; tail -2 gpurun_out/launches.csv
