python -c "from tools.build_native import build_all; build_all()"
for d in 1 0 1; do XK_DEFER_D2H=$d python bench.py --no-cpu-baseline --steps 3 > gpurun_out/b_$d.json 2>/dev/null; python -c "
import json;d=json.load(open('gpurun_out/b_$d.json'));print('defer=$d', round(d['value'],2), round(d['e2e']['value'],2))"; done
BLAS3=1 bash tools/gpu_iter.sh
