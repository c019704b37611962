#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:trxm_base -s 3 -c 1 -f -o gpurun_out/trsm_base python tools/trsm_panel.py > gpurun_out/trsm_ncu.log 2>&1
ls -la gpurun_out/trsm_base.ncu-rep
