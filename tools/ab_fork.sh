#!/bin/bash
export PYTHONUNBUFFERED=1
for F in 0 1 2 0 1 2; do
  BETTY_REG_FORK=$F timeout -s KILL 600 python bench.py --steps 20 --cpu-sample-outputs 16 > gpurun_out/fork.log 2>&1
  python - <<PY
import json
d=json.loads(open('gpurun_out/fork.log').read().strip().splitlines()[-1])
print('fork $F ms/step', round(d['ms_per_step'],4), {k: round(v,3) for k,v in d['roofline']['other_sites_ms_per_step'].items()})
PY
done
BETTY_REG_FORK=1 timeout -s KILL 600 python bench.py --sim-world 8 --steps 20 --cpu-sample-outputs 16 | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('N8 fork1', d['ms_per_step'])"
BETTY_REG_FORK=2 timeout -s KILL 600 python bench.py --sim-world 8 --steps 20 --cpu-sample-outputs 16 | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('N8 fork2', d['ms_per_step'])"
