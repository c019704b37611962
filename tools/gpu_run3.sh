#!/bin/bash
# round-2 A/Bs: TRSM diagonal-group ramp and update-window depth; GEMM snake raster (DRAM
# bytes + speed); planner-model fidelity with the grouped task-rate probe
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
for cfg in "base" "XK_DIAG_RAMP=1" "XK_TRSM_DMUL=2" "XK_TRSM_DMUL=4" "XK_DIAG_RAMP=1 XK_TRSM_DMUL=2"; do
  if [ "$cfg" = base ]; then envs=""; else envs="$cfg"; fi
  env $envs ROUTINES="dtrsm" timeout 600 python tools/bench_blas3.py 2>&1 | tail -1 | sed "s/^/$cfg /" >> gpurun_out/trsm_ab.txt
done
for sn in 1 0; do
  XK_SNAKE=$sn timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct \
      --clock-control none -k regex:dgemm_tma -s 40 -c 1 --csv \
      python bench.py --size 32768 --tile 4096 --steps 1 --warmup 1 --no-cpu-baseline --host-probe-mib 256 \
      > gpurun_out/snake_${sn}_ncu.csv 2> gpurun_out/snake_${sn}_ncu.err
  XK_SNAKE=$sn timeout 600 python tools/gemm_ab.py > gpurun_out/snake_${sn}_ab.json 2>&1
done
for sn in 1 0; do XK_SNAKE=$sn timeout 600 python tools/gemm_ab.py >> gpurun_out/snake_${sn}_ab.json 2>&1; done
CASES="dgemm:16384:2048 dgemm:32768:4096 dtrsm:32768:2048 dsyr2k:32768:2048" timeout 900 python tools/model_fidelity.py > gpurun_out/fidelity2.jsonl 2> gpurun_out/fidelity2.err
