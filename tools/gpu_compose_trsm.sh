#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
for G in 1 8; do for N in 16384 32768; do
  ROUTINE=trsm G=$G N=$N T=2048 timeout 900 python tools/compose.py 2>/dev/null | tail -1 | tee gpurun_out/compose_trsm_n${N}_g${G}.json
done; done
