#!/bin/bash
export PYTHONUNBUFFERED=1
timeout -s KILL 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_c5.py -x -q -k "mean3 or c5 or step" > gpurun_out/q9_tests.log 2>&1; echo "tests rc=$?"; tail -1 gpurun_out/q9_tests.log
for i in 1 2; do
timeout -s KILL 600 python bench.py --config C5 --scale 0.1 --steps 10 --cpu-sample-outputs 16 > gpurun_out/q9.log 2>&1
python -c "
import json; d=json.loads(open('gpurun_out/q9.log').read().strip().splitlines()[-1]); print('C5@0.1 ms', d['ms_per_step'])"
done
