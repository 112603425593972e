#!/bin/bash
# quick GPU check: REG/plan parity tests + C3 bench + per-rank study at N=8
export PYTHONUNBUFFERED=1
timeout -s KILL 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -x -q -k "reg or plan or step" > gpurun_out/quick_tests.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/quick_tests.log
for N in 1 8; do
  timeout -s KILL 600 python bench.py --sim-world $N --steps 20 --cpu-sample-outputs 16 > gpurun_out/q_$N.log 2>&1; echo "N=$N rc=$?"
  python - <<PY
import json
d=json.loads(open('gpurun_out/q_$N.log').read().strip().splitlines()[-1])
print('N=$N ms/step', round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['roofline']['other_sites_ms_per_step'].items()})
PY
done
