#!/bin/bash
# DRAM traffic and speed of the grouped T=4096 DGEMM launch per raster group (XK_GROUP_M):
# ncu dram bytes + duration of one 16-task grouped launch of the bench workload, then the
# data-on-device A/B (no profiler) at T=4096.
mkdir -p gpurun_out
for gm in ${GMS:-8 16 32 64}; do
  XK_GROUP_M=$gm timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct \
      --clock-control none -k regex:dgemm_tma -s 40 -c 1 --csv \
      python bench.py --size 32768 --tile 4096 --steps 1 --warmup 1 --no-cpu-baseline --host-probe-mib 256 \
      > gpurun_out/groupm_${gm}_ncu.csv 2> gpurun_out/groupm_${gm}_ncu.err
  XK_GROUP_M=$gm TILES=4096 timeout 600 python tools/gemm_ab.py > gpurun_out/groupm_${gm}_ab.json 2>&1
  tail -1 gpurun_out/groupm_${gm}_ab.json
done
