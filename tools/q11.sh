#!/bin/bash
export PYTHONUNBUFFERED=1
timeout -s KILL 600 python -m pytest tests/test_gpu_gemm.py -x -q > gpurun_out/q11_tests.log 2>&1; echo "tests rc=$?"; tail -1 gpurun_out/q11_tests.log
for i in 1 2; do
timeout -s KILL 600 python bench.py --steps 20 --cpu-sample-outputs 16 --e2e-steps 3 > gpurun_out/q11.log 2>&1
python - <<PY
import json
d=json.loads(open('gpurun_out/q11.log').read().strip().splitlines()[-1])
print('ms/step', round(d['ms_per_step'],4), {k: round(v,3) for k,v in d['roofline']['other_sites_ms_per_step'].items()})
PY
done
bash tools/launches.sh q11 > gpurun_out/q11_launch.txt 2>&1; grep -E "tc_row|one step" gpurun_out/q11_launch.txt
