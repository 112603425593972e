#!/bin/bash
export PYTHONUNBUFFERED=1
for L in l2 gid; do for G in 1 0; do
  BETTY_AGG_G4=$G timeout -s KILL 600 python bench.py --feat-layout $L --steps 10 --cpu-sample-outputs 16 > gpurun_out/l2res_$L$G.log 2>&1
  python - <<PY
import json
d=json.loads(open('gpurun_out/l2res_$L$G.log').read().strip().splitlines()[-1])
print('$L g4=$G ms/step', round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['roofline']['other_sites_ms_per_step'].items()})
PY
done; done
