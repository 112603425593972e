#!/bin/bash
export PYTHONUNBUFFERED=1
for V in base f2r4 f8r4 f4r2 f4r6 base; do
  if [ $V = base ]; then L=""; else L="$PWD/paper_conf_asplos_yangzd023_b200/build_var/$V/libbetty.so"; fi
  BETTY_LIB_PATH=$L timeout -s KILL 600 python bench.py --steps 20 --cpu-sample-outputs 16 --e2e-steps 3 > gpurun_out/ex.log 2>&1
  python - <<PY
import json
d=json.loads(open('gpurun_out/ex.log').read().strip().splitlines()[-1])
print('$V ms/step', round(d['ms_per_step'],4), 'extract', round(d['roofline']['other_sites_ms_per_step']['extract'],4))
PY
done
