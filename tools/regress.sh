#!/bin/bash
# Quick performance regression sweep over the presets (run under gpurun): one short bench line per
# config (C1-C4, plus the 8-rank share of C3), ms/step and the site times -- catches a change that
# helps one workload and hurts another (e.g. the full-neighbourhood C2).
export PYTHONUNBUFFERED=1
for C in C1 C2 C3 C4; do
  S=20; [ $C = C4 ] && S=3
  timeout -s KILL 600 python bench.py --config $C --steps $S --no-fp32 --cpu-sample-outputs 16 > gpurun_out/regress_$C.log 2>&1
  tail -1 gpurun_out/regress_$C.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d.get('roofline') or {}; print('$C', round(d['ms_per_step'],3), {k: round(v,3) for k,v in (r.get('other_sites_ms_per_step') or {}).items()})"
done
timeout -s KILL 600 python bench.py --sim-world 8 --steps 20 --no-fp32 --cpu-sample-outputs 16 > gpurun_out/regress_sim8.log 2>&1
tail -1 gpurun_out/regress_sim8.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C3 sim8', round(d['ms_per_step'],4))"
