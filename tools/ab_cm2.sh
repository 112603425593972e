#!/bin/bash
export PYTHONUNBUFFERED=1
for V in 0 1 2 3; do
  BETTY_CSC_MEAN_VAR=$V timeout -s KILL 600 python bench.py --config C5 --scale 0.1 --steps 10 --cpu-sample-outputs 16 > gpurun_out/abcm2.log 2>&1
  python - <<PY
import json
d=json.loads(open('gpurun_out/abcm2.log').read().strip().splitlines()[-1])
print('var $V ms/step', round(d['ms_per_step'],3))
PY
done
