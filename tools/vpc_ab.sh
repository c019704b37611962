#!/bin/bash
# A/B of the base kernel's vectors per CTA (XK_VPC) on the TRSM panel driver and DTRSM
mkdir -p gpurun_out
for V in ${VPCS:-128 256}; do
  touch paper_conf_sc_gautierl21_b200/csrc/kernels/trxm_tile.cu
  NVCC_APPEND_FLAGS="-DXK_VPC=$V" python -c "from tools.build_native import build_xk; build_xk()" || exit 1
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/vpc$V.csv -k regex:trxm_base python tools/trsm_panel.py > /dev/null 2>&1
  python - $V <<'PY'
import csv, sys
rows = list(csv.reader(open("gpurun_out/vpc%s.csv" % sys.argv[1])))
h = [r for r in rows if "Metric Value" in r][0]
vals = [float(dict(zip(h, r))["Metric Value"].replace(",", "")) for r in rows if len(r) == len(h) and r is not h and dict(zip(h, r)).get("Metric Name") == "gpu__time_duration.sum"]
print("VPC=%s base launches %d avg %.1f (ncu unit)" % (sys.argv[1], len(vals), sum(vals) / len(vals)))
PY
  ROUTINES="dtrsm" timeout 600 python tools/bench_blas3.py 2>/dev/null | tail -1
done
