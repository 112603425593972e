#!/bin/bash
# A/B of the layer-0 aggregation kernels on the bench workload + ncu of the g4 kernel
export PYTHONUNBUFFERED=1
TAG=${1:-ab}
for G in 0 1; do
  BETTY_AGG_G4=$G timeout -s KILL 600 python bench.py --steps 10 > gpurun_out/bench_${TAG}_g4$G.log 2>&1
  python - <<PY
import json
d=json.loads(open('gpurun_out/bench_${TAG}_g4$G.log').read().strip().splitlines()[-1])
print('G4=$G ms/step', round(d['ms_per_step'],3), 'frac', round(d['roofline']['frac'],3), {k: round(v,3) for k,v in d['roofline']['other_sites_ms_per_step'].items()})
PY
done
bash tools/prof_full.sh ${TAG} "k_agg_mean" 1 > /dev/null 2>&1
python tools/ncu_table.py gpurun_out/full_${TAG}_raw.csv
