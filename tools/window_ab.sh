#!/bin/bash
# A/B of the planner's prefetch window W on one GPU (e2e host-resident DGEMM + DTRSM)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
for W in 2 4 2 4; do
  XK_WINDOW=$W timeout 900 python bench.py --steps 3 --warmup 2 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('W=$W value %.2f e2e %.2f' % (d['value'], d['e2e']['value']))"
done
for W in 2 4; do XK_WINDOW=$W ROUTINES="dtrsm dsyrk" timeout 600 python tools/bench_blas3.py 2>/dev/null | tail -1 | sed "s/^/W=$W /"; done
