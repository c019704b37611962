#!/bin/bash
# rank mode (one process per GPU) under torchrun on the one-GPU box: both ranks share the
# device (gloo for the host-side barriers; NCCL refuses two ranks on one GPU)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
N=${N:-16384}; T=${T:-2048}; W=${W:-2}
XK_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node $W \
  --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus $W --size $N --tile $T --steps 2 --warmup 1 \
  > gpurun_out/rank_bench_w$W.json 2> gpurun_out/rank_bench_w$W.err
tail -5 gpurun_out/rank_bench_w$W.err; cat gpurun_out/rank_bench_w$W.json
timeout 600 python bench.py --n $N --tile $T --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/bench_w1.json 2> gpurun_out/bench_w1.err
tail -3 gpurun_out/bench_w1.err; cat gpurun_out/bench_w1.json
