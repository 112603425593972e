#!/bin/bash
export PYTHONUNBUFFERED=1
timeout -s KILL 600 python -m pytest tests/test_gpu_parity.py -x -q -k "step or plan" > gpurun_out/prio_tests.log 2>&1; echo "tests rc=$?"; tail -1 gpurun_out/prio_tests.log
run() {
  env $1 timeout -s KILL 600 python bench.py $2 --steps 20 --cpu-sample-outputs 16 > gpurun_out/prio.log 2>&1
  python - <<PY
import json
d=json.loads(open('gpurun_out/prio.log').read().strip().splitlines()[-1])
print('$1 $2 ms/step', round(d['ms_per_step'],4), {k: round(v,3) for k,v in d['roofline']['other_sites_ms_per_step'].items()})
PY
}
run X=1 ""
run BETTY_NO_NODE_PRIORITY=1 ""
run X=1 ""
run BETTY_NO_NODE_PRIORITY=1 ""
run X=1 "--sim-world 8"
run BETTY_NO_NODE_PRIORITY=1 "--sim-world 8"
