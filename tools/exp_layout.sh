#!/bin/bash
# A/B of the feature-table row layout (gid vs owner) on C3 (run under gpurun).
export PYTHONUNBUFFERED=1
for L in owner gid; do
  timeout -s KILL 600 python bench.py --feat-layout $L --cpu-sample-outputs 64 > gpurun_out/layout_$L.log 2>&1; echo "$L rc=$?"
  python - <<PY
import json
d=json.loads(open('gpurun_out/layout_$L.log').read().strip().splitlines()[-1])
print('$L ms/step', d['ms_per_step'], 'Gedges/s', d['value']/1e9, 'frac', d['roofline']['frac'], {k: round(v,3) for k,v in d['roofline']['other_sites_ms_per_step'].items()})
PY
  grep "feature layout" gpurun_out/layout_$L.log
done
