#!/bin/bash
# Study: community-contiguous node ids (locality upper bound) x L1-allocating gathers
export PYTHONUNBUFFERED=1
run() { # name, env, args
  env $2 timeout -s KILL 600 python bench.py $3 --steps 10 --cpu-sample-outputs 16 > gpurun_out/loc_$1.log 2>&1
  python - <<PY
import json
d=json.loads(open('gpurun_out/loc_$1.log').read().strip().splitlines()[-1])
print('$1 ms/step', round(d['ms_per_step'],3), 'edges', d['edges_per_step'], {k: round(v,3) for k,v in d['roofline']['other_sites_ms_per_step'].items()})
PY
}
run comm_g4 "BETTY_AGG_G4=1" "--input-order community"
run comm_ca "BETTY_AGG_G4=0 BETTY_AGG_CA=1" "--input-order community"
run comm_bulk "BETTY_AGG_G4=0" "--input-order community"
run rand_ca "BETTY_AGG_G4=0 BETTY_AGG_CA=1" ""
