#!/bin/bash
export PYTHONUNBUFFERED=1
TAG=${1:-r01i}
timeout -s KILL 900 python bench.py > gpurun_out/bench_C3_${TAG}.log 2>&1; echo "C3 rc=$?"; tail -1 gpurun_out/bench_C3_${TAG}.log > gpurun_out/bench_C3_${TAG}.jsonl
timeout -s KILL 1500 python bench.py --config C5 --steps 5 > gpurun_out/bench_C5_${TAG}.log 2>&1; echo "C5 rc=$?"; tail -1 gpurun_out/bench_C5_${TAG}.log > gpurun_out/bench_C5_${TAG}.jsonl
BETTY_BENCH_ONE_GPU=1 timeout -s KILL 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 5 --warmup 3 > gpurun_out/bench2_${TAG}.log 2>&1; echo "2-rank rc=$?"
for f in gpurun_out/bench_C3_${TAG}.jsonl gpurun_out/bench_C5_${TAG}.jsonl; do
python - <<PY
import json
d=json.loads(open('$f').read())
print('$f', 'ms/step', round(d['ms_per_step'],3), 'Gedges/s', round(d['value']/1e9,3), 'frac', d['roofline']['frac'], 'e2e', round(d['e2e']['value']/1e9,3), d['e2e'].get('input_buffers'))
PY
done
tail -c 300 gpurun_out/bench2_${TAG}.log
