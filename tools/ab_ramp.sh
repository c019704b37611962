python -c "from tools.build_native import build_all; build_all()"
for r in 1 2 4 8 1 4; do XK_RAMP=$r python bench.py --no-cpu-baseline --steps 3 > gpurun_out/b_$r.json 2>/dev/null; python -c "
import json;d=json.load(open('gpurun_out/b_$r.json'));print('ramp=$r', round(d['value'],2), round(d['e2e']['value'],2))"; done
for r in 1 4; do XK_RAMP=$r python bench.py --no-cpu-baseline --steps 3 --tile 2048 > gpurun_out/b_$r.json 2>/dev/null; python -c "
import json;d=json.load(open('gpurun_out/b_$r.json'));print('T2048 ramp=$r', round(d['value'],2), round(d['e2e']['value'],2))"; done
