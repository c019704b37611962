#!/bin/bash
# TRSM/TRMM base kernel: vectors per CTA (XK_NVB 64 = default, 32) -- per-launch time from the
# ncu launch list of a data-on-device DTRSM N=16384 (tools/trsm_panel.py), then DTRSM throughput
mkdir -p gpurun_out
build() { python -c "from tools.build_native import build_xk; build_xk(force=True)" || exit 1; }
for nvb in 64 32; do
  XK_NVCC_FLAGS="-DXK_NVB=$nvb" build
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:trxm_base --csv --log-file gpurun_out/nvb_${nvb}_launches.csv python tools/trsm_panel.py > /dev/null 2>&1
  python - $nvb <<'PY'
import csv, sys
nvb = sys.argv[1]
rows = [r for r in csv.reader(open("gpurun_out/nvb_%s_launches.csv" % nvb)) if len(r) > 5]
h = rows[0]; vi = h.index("Metric Value")
v = [float(r[vi].replace(",", "")) for r in rows[1:]]
print("NVB=%s trxm_base launches %d avg %.2f us" % (nvb, len(v), sum(v) / len(v) / 1e3))
PY
  ROUTINES="dtrsm" timeout 900 python tools/bench_blas3.py 2>&1 | tail -1 | sed "s/^/NVB=$nvb | /"
done
XK_NVCC_FLAGS="" build
