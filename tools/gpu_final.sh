#!/bin/bash
# end-of-round verification + evidence: GPU suite, smoke, bench (both arms), ncu launch list
# and a full capture of the grouped T=4096 launch (the bench's dominant kernel), model fidelity,
# BLAS-3 table, BASELINE configs[4] on one GPU
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -5 > gpurun_out/gpu_tests.txt
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1 > gpurun_out/smoke.txt
python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
CMD="python bench.py --size 32768 --tile 4096 --steps 1 --warmup 1 --no-cpu-baseline --host-probe-mib 256"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file gpurun_out/launches.csv $CMD > gpurun_out/ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dgemm_tma -s 40 -c 1 -f -o gpurun_out/tile_full $CMD > gpurun_out/ncu_full.log 2>&1
python tools/ncu_tile_json.py gpurun_out/tile_full.ncu-rep 4096 16 "ncu --set full --clock-control none -k regex:dgemm_tma -s 40 -c 1 $CMD" > gpurun_out/dgemm_tile_ncu.json
ncu -i gpurun_out/tile_full.ncu-rep --page details --csv > gpurun_out/tile_full_details.csv 2>/dev/null
timeout 900 python tools/model_fidelity.py > gpurun_out/fidelity.jsonl 2> gpurun_out/fidelity.err
timeout 900 python tools/bench_blas3.py > gpurun_out/blas3.txt 2>&1
timeout 1500 python tools/config5.py > gpurun_out/config5.txt 2>&1
