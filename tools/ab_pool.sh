#!/bin/bash
export PYTHONUNBUFFERED=1
timeout -s KILL 600 python -m pytest tests/test_gpu_parity.py -x -q -k "pool" > gpurun_out/tests_pool.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/tests_pool.log
for V in "X=1" "BETTY_POOL_POS8=1"; do
  env $V timeout -s KILL 900 python bench.py --config C4 --steps 3 --warmup 3 > gpurun_out/bench_pool.log 2>&1; echo "$V rc=$?"
  python -c "
import json; d=json.loads(open('gpurun_out/bench_pool.log').read().strip().splitlines()[-1]); print('$V C4 ms', d['ms_per_step'], 'K', d['config']['K'], 'Gedges/s', d['value']/1e9)"
done
