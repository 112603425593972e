#!/bin/bash
# A/B of the layer-0 aggregation variants on the bench workload
export PYTHONUNBUFFERED=1
TAG=${1:-ab}
run() {
  env $1 timeout -s KILL 600 python bench.py --steps 10 > gpurun_out/bench_${TAG}_$2.log 2>&1
  python - <<PY
import json
d=json.loads(open('gpurun_out/bench_${TAG}_$2.log').read().strip().splitlines()[-1])
print('$2 ms/step', round(d['ms_per_step'],3), 'frac', round(d['roofline']['frac'],3), {k: round(v,3) for k,v in d['roofline']['other_sites_ms_per_step'].items()})
PY
}
run BETTY_AGG_G4=1 g4
run BETTY_AGG_G4=0 bulk
run "BETTY_AGG_G4=0 BETTY_AGG_NOBULK=1" lanes
