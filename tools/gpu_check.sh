#!/bin/bash
# GPU round trip: parity tests, bench, launch list of one step (run under gpurun).
export PYTHONUNBUFFERED=1
TAG=${1:-dev}
timeout -s KILL 900 python -m pytest tests -m gpu -x -q > gpurun_out/tests_${TAG}.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/tests_${TAG}.log
timeout -s KILL 600 python bench.py > gpurun_out/bench_${TAG}.log 2>&1; echo "bench rc=$?"
python - <<PY
import json
d=json.loads(open('gpurun_out/bench_${TAG}.log').read().strip().splitlines()[-1])
print('ms/step', d['ms_per_step'], 'Gedges/s', d['value']/1e9, 'frac', d['roofline']['frac'], {k: round(v,3) for k,v in d['roofline']['other_sites_ms_per_step'].items()})
PY
timeout -s KILL 600 ncu --profile-from-start off --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
  --log-file gpurun_out/launches_${TAG}.csv python tools/prof_step.py > /dev/null 2>&1; echo "launches rc=$?"
