#!/bin/bash
# the driver's 8-GPU bench command, in rank mode with 8 processes sharing the one B200
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
XK_DIST_BACKEND=gloo timeout 1500 python -m torch.distributed.run --nnodes=1 --nproc-per-node 8 \
  --master-addr 127.0.0.1 --master-port 29541 bench.py --gpus 8 --steps 2 --warmup 1 --no-cpu-baseline \
  > gpurun_out/rank_bench_w8.json 2> gpurun_out/rank_bench_w8.err
echo "rc=$?" >> gpurun_out/rank_bench_w8.err
