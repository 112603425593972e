#!/bin/bash
export PYTHONUNBUFFERED=1
timeout -s KILL 600 python -m pytest tests/test_gpu_gemm.py tests/test_gpu_parity.py -x -q > gpurun_out/es_tests.log 2>&1; echo "tests rc=$?"; tail -1 gpurun_out/es_tests.log
for V in 2 0 2 0; do
  BETTY_GEMM_ESLOTS=$V timeout -s KILL 600 python bench.py --steps 20 --cpu-sample-outputs 16 > gpurun_out/es.log 2>&1
  python - <<PY
import json
d=json.loads(open('gpurun_out/es.log').read().strip().splitlines()[-1])
print('eslots $V ms/step', round(d['ms_per_step'],4))
PY
done
BETTY_GEMM_ESLOTS=0 timeout -s KILL 600 python bench.py --config C5 --scale 0.1 --steps 10 --cpu-sample-outputs 16 | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('C5@0.1', d['ms_per_step'])"
