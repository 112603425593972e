#!/bin/bash
# ab.sh "VARIANTS" BENCH_ARGS...: one bench line per libbetty variant (build_var/NAME, "base" = the
# in-tree build), printing ms/step and the probed sites.  VARIANTS space-separated; REPS repeats.
export PYTHONUNBUFFERED=1
VARS=$1; shift
for r in $(seq ${REPS:-1}); do
for V in $VARS; do
  if [ $V = base ]; then L=""; else L="$PWD/paper_conf_asplos_yangzd023_b200/build_var/$V/libbetty.so"; fi
  BETTY_LIB_PATH=$L timeout -s KILL 900 python bench.py --cpu-sample-outputs 0 --e2e-steps 2 "$@" > gpurun_out/ab_$V.log 2>&1
  python - "$V" <<'PY'
import json, sys
v = sys.argv[1]
try:
    d = json.loads(open(f'gpurun_out/ab_{v}.log').read().strip().splitlines()[-1])
    st = {k: round(x, 3) for k, x in d['roofline']['other_sites_ms_per_step'].items()}
    print(f"{v:10s} ms/step {d['ms_per_step']:.4f} {st}")
except Exception as e:
    print(v, 'FAILED', open(f'gpurun_out/ab_{v}.log').read()[-600:])
PY
done
done
