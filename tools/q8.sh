#!/bin/bash
export PYTHONUNBUFFERED=1
timeout -s KILL 900 python -m pytest tests/test_gpu_parity.py -x -q -k "pool" > gpurun_out/q8_tests.log 2>&1; echo "tests rc=$?"; tail -1 gpurun_out/q8_tests.log
for i in 1 2; do
timeout -s KILL 900 python bench.py --config C4 --steps 5 --warmup 3 --cpu-sample-outputs 1 > gpurun_out/q8.log 2>&1
python -c "
import json; d=json.loads(open('gpurun_out/q8.log').read().strip().splitlines()[-1]); print('C4 ms', d['ms_per_step'])"
done
