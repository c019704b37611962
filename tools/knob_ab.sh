#!/bin/bash
# A/B of executor/kernel knobs on the bench workload (value = data-on-device DGEMM N=32768 T=4096)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
run() { env "$@" timeout 600 python bench.py --steps 3 --warmup 2 --no-cpu-baseline --no-e2e 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$* value %.3f frac %.4f' % (d['value'], d['roofline']['frac']))"; }
for rep in 1 2; do
  run XK_GROUP_M=16
  run XK_GROUP_M=8
  run XK_GROUP_M=32
  run XK_BATCH=32
  run XK_KSTREAMS=3
done
