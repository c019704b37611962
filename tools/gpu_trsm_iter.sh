#!/bin/bash
# TRSM/TRMM diagonal-tile work: parity, launch list of the panel driver, BLAS-3 throughput
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 python -m pytest tests/test_gpu_blas3.py tests/test_gpu_fuzz.py tests/test_gpu_rank.py -x -q -k "not freivalds" 2>&1 | tail -4 | tee gpurun_out/trsm_tests.txt
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/trsm_launches.csv python tools/trsm_panel.py > /dev/null 2>&1
python - <<'PY' | tee gpurun_out/trsm_launch_summary.txt
import csv, collections
rows = list(csv.reader(open("gpurun_out/trsm_launches.csv")))
h = None; agg = collections.defaultdict(lambda: [0, 0.0])
for r in rows:
    if "Kernel Name" in r: h = r; continue
    if h and len(r) == len(h):
        d = dict(zip(h, r))
        if d.get("Metric Name") == "gpu__time_duration.sum":
            k = d["Kernel Name"].split("(")[0].split("<")[0]
            v = float(d["Metric Value"].replace(",", ""))
            u = d.get("Metric Unit", "")
            v = v / 1000.0 if u == "nsecond" else v * (1000.0 if u == "msecond" else 1.0)
            agg[k][0] += 1; agg[k][1] += v
tot = sum(a[1] for a in agg.values())
for k, (n, us) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
    print("%-40s %6d launches %10.1f us total %8.2f us avg  %5.1f%%" % (k[-40:], n, us, us / n, 100 * us / tot))
PY
ROUTINES=${ROUTINES:-} timeout 900 python tools/bench_blas3.py > gpurun_out/blas3.json 2> gpurun_out/blas3.err; tail -40 gpurun_out/blas3.json
