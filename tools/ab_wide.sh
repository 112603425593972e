#!/bin/bash
export PYTHONUNBUFFERED=1
timeout -s KILL 900 python -m pytest tests -m gpu -x -q > gpurun_out/wide_tests.log 2>&1; echo "tests auto rc=$?"; tail -1 gpurun_out/wide_tests.log
BETTY_GEMM_WIDE=1 timeout -s KILL 900 python -m pytest tests/test_gpu_gemm.py tests/test_gpu_parity.py tests/test_gpu_c5.py -x -q > gpurun_out/wide_tests1.log 2>&1; echo "tests forced rc=$?"; tail -1 gpurun_out/wide_tests1.log
for V in 0 -1 1 0 -1 1; do
  BETTY_GEMM_WIDE=$V timeout -s KILL 600 python bench.py --steps 20 --cpu-sample-outputs 16 > gpurun_out/wide.log 2>&1
  python - <<PY
import json
d=json.loads(open('gpurun_out/wide.log').read().strip().splitlines()[-1])
print('wide $V ms/step', round(d['ms_per_step'],4), {k: round(v,3) for k,v in d['roofline']['other_sites_ms_per_step'].items()})
PY
done
