#!/bin/bash
export PYTHONUNBUFFERED=1
timeout -s KILL 600 python -m pytest tests/test_gpu_gemm.py tests/test_gpu_c5.py tests/test_gpu_parity.py -x -q > gpurun_out/q2_tests.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/q2_tests.log
for A in "--config C5 --scale 0.1" "--config C3"; do
  timeout -s KILL 600 python bench.py $A --steps 10 --cpu-sample-outputs 16 > gpurun_out/q2.log 2>&1
  python - <<PY
import json
d=json.loads(open('gpurun_out/q2.log').read().strip().splitlines()[-1])
print('$A ms/step', round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['roofline']['other_sites_ms_per_step'].items()})
PY
done
