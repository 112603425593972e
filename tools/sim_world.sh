#!/bin/bash
# Per-rank step time of rank 0's share at N = 2, 4, 8 (one GPU; study, not bench values) + launch list at N=8
export PYTHONUNBUFFERED=1
for N in 2 4 8; do
  timeout -s KILL 600 python bench.py --sim-world $N --steps 10 --cpu-sample-outputs 16 > gpurun_out/sim_$N.log 2>&1; echo "N=$N rc=$?"
  python - <<PY
import json
d=json.loads(open('gpurun_out/sim_$N.log').read().strip().splitlines()[-1])
print('N=$N ms/step', round(d['ms_per_step'],3), 'mb/rank', d['config']['micro_batches_per_rank'], {k: round(v,3) for k,v in d['roofline']['other_sites_ms_per_step'].items()})
PY
done
