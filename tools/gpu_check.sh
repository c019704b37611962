#!/bin/bash
# GPU pass during development: build, all -m gpu tests (or PYTEST_K subset), smoke, a short bench
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout ${TEST_TIMEOUT:-1500} python -m pytest tests -m gpu -x -q ${PYTEST_K:+-k "$PYTEST_K"} 2>&1 | tail -30 > gpurun_out/gpu_tests.txt; tail -3 gpurun_out/gpu_tests.txt
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 900 python bench.py ${BENCH_ARGS:---steps 5 --warmup 3} > gpurun_out/bench.json 2> gpurun_out/bench.err; tail -2 gpurun_out/bench.err; cat gpurun_out/bench.json
