#!/bin/bash
export PYTHONUNBUFFERED=1
timeout -s KILL 600 python bench.py > gpurun_out/q10.log 2>&1; echo "rc=$?"
python - <<PY
import json
d=json.loads(open('gpurun_out/q10.log').read().strip().splitlines()[-1])
print('ms/step', d['ms_per_step'], 'e2e', d['e2e'])
PY
grep -i "e2e:" gpurun_out/q10.log
timeout -s KILL 900 python bench.py --config C4 --steps 3 --cpu-sample-outputs 1 > gpurun_out/q10b.log 2>&1; echo "c4 rc=$?"
python - <<PY
import json
d=json.loads(open('gpurun_out/q10b.log').read().strip().splitlines()[-1])
print('C4 ms/step', d['ms_per_step'], 'e2e', d['e2e'])
PY
grep -i "e2e:" gpurun_out/q10b.log
