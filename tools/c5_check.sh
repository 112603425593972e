#!/bin/bash
export PYTHONUNBUFFERED=1
timeout -s KILL 900 python -m pytest tests -m gpu -x -q > gpurun_out/tests_cm.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/tests_cm.log
timeout -s KILL 1200 python bench.py --config C5 --steps 5 --warmup 3 > gpurun_out/c5_cm.log 2> gpurun_out/c5_cm.err; echo "c5 rc=$?"
python - <<PY
import json
d=json.loads(open('gpurun_out/c5_cm.log').read().strip().splitlines()[-1])
print('C5 ms/step', d['ms_per_step'], 'Gedges/s', d['value']/1e9, 'frac', d['roofline']['frac'], {k: round(v,3) for k,v in d['roofline']['other_sites_ms_per_step'].items()})
PY
