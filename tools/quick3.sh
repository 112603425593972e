#!/bin/bash
export PYTHONUNBUFFERED=1
python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" 2>&1 | tail -1
for A in "" "--no-reg" "" "--no-reg"; do
  timeout -s KILL 600 python bench.py $A --steps 20 --cpu-sample-outputs 16 > gpurun_out/q3.log 2>&1
  python - <<PY
import json
d=json.loads(open('gpurun_out/q3.log').read().strip().splitlines()[-1])
print('$A ms/step', round(d['ms_per_step'],4))
PY
done
