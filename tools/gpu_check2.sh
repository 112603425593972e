#!/bin/bash
# GPU round trip: parity tests, bench (C3), and the 2-rank bench path on one GPU (run under gpurun).
export PYTHONUNBUFFERED=1
TAG=${1:-dev}
timeout -s KILL 900 python -m pytest tests -m gpu -x -q > gpurun_out/tests_${TAG}.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/tests_${TAG}.log
timeout -s KILL 600 python bench.py > gpurun_out/bench_${TAG}.log 2>&1; echo "bench rc=$?"
python - <<PY
import json
d=json.loads(open('gpurun_out/bench_${TAG}.log').read().strip().splitlines()[-1])
print('ms/step', d['ms_per_step'], 'Gedges/s', d['value']/1e9, 'frac', d['roofline']['frac'], {k: round(v,3) for k,v in d['roofline']['other_sites_ms_per_step'].items()})
PY
BETTY_BENCH_ONE_GPU=1 timeout -s KILL 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 5 --warmup 3 > gpurun_out/bench2_${TAG}.log 2>&1; echo "bench 2-rank rc=$?"; tail -c 1500 gpurun_out/bench2_${TAG}.log
