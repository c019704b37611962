python -c "from tools.build_native import build_all; build_all()"
for r in 8 16 32 8; do XK_RAMP=$r python bench.py --no-cpu-baseline --steps 3 > gpurun_out/b_$r.json 2>/dev/null; python -c "
import json;d=json.load(open('gpurun_out/b_$r.json'));print('ramp=$r', round(d['value'],2), round(d['e2e']['value'],2))"; done
ROUTINE=dgemm T=4096 python tools/trace_routine.py > gpurun_out/tr.log 2>&1; tail -1 gpurun_out/tr.log | cut -c1-2500
