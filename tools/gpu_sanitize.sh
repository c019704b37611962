#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
for t in memcheck racecheck synccheck; do
  echo "== $t"; timeout 900 compute-sanitizer --tool $t --print-limit 10 python tools/sanitize_small.py 2>&1 | tail -3
done | tee gpurun_out/sanitizer.txt
