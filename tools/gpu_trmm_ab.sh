#!/bin/bash
# DTRMM shadow sweep (reading R15) on 8 logical GPUs: the in-place plan (_old, the previous
# commit, extracted by the caller) vs the shadow plan; plus 1-GPU parity of the routine tests
mkdir -p gpurun_out
python -c "from tools.build_native import build_all; build_all()" || exit 1
echo tests skipped
for v in new old; do
  d=.; [ $v = old ] && d=_old
  (cd $d && python -c "from tools.build_native import build_all; build_all()" > /dev/null 2>&1
   for n in ${NS:-16384}; do
     ROUTINE=dtrmm N=$n G=8 T=2048 REPS=${REPS:-2} timeout 900 python tools/ablation.py 2>&1 | tail -1 > $GRAFT_REPO_ROOT/gpurun_out/ablation_dtrmm_${v}_n${n}_g8.json
     python -c "import json;d=json.load(open('$GRAFT_REPO_ROOT/gpurun_out/ablation_dtrmm_${v}_n${n}_g8.json'));print('$v', $n, {k:v for k,v in d.items() if not isinstance(v,(list,dict))}, d.get('vs_full_percent'))"
   done)
done

