#!/bin/bash
export PYTHONUNBUFFERED=1
timeout -s KILL 900 python -m pytest tests -m gpu -x -q -k "c5 or step or invariant or c2 or sage" > gpurun_out/tests_cmg.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/tests_cmg.log
for V in "X=1" "BETTY_CSC_MEAN_WARP=1"; do
  env $V timeout -s KILL 600 python bench.py --config C5 --scale 0.1 --steps 10 --cpu-sample-outputs 16 > gpurun_out/abcm.log 2>&1
  python - <<PY
import json
d=json.loads(open('gpurun_out/abcm.log').read().strip().splitlines()[-1])
print('$V ms/step', round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['roofline']['other_sites_ms_per_step'].items()})
PY
done
