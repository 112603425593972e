#!/bin/bash
# layer-0 aggregation under other gather4 pipeline shapes (tools/build_g4_variants.sh builds them)
export PYTHONUNBUFFERED=1
for V in base ${SWEEP:-m8 m32 cl32 cl128}; do
  if [ $V = base ]; then L=""; else L="$PWD/paper_conf_asplos_yangzd023_b200/build_var/$V/libbetty.so"; fi
  BETTY_LIB_PATH=$L timeout -s KILL 600 python bench.py --steps 20 --cpu-sample-outputs 0 --e2e-steps 2 --no-fp32 > gpurun_out/g4.log 2>&1
  python - <<PY
import json
d=json.loads(open('gpurun_out/g4.log').read().strip().splitlines()[-1])
print('$V ms/step', round(d['ms_per_step'],4), 'agg_l0', round(d['roofline']['other_sites_ms_per_step']['agg_l0'],4))
PY
done
