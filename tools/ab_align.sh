export PYTHONUNBUFFERED=1
for A in 0 256; do for G in 1 0; do
  BETTY_AGG_G4=$G timeout -s KILL 600 python bench.py --steps 10 --feat-align $A > gpurun_out/bench_al_${A}_$G.log 2>&1
  python -c "
import json; d=json.loads(open('gpurun_out/bench_al_${A}_$G.log').read().strip().splitlines()[-1]); print('align $A g4 $G ms', round(d['ms_per_step'],3), 'frac', round(d['roofline']['frac'],3), {k: round(v,3) for k,v in d['roofline']['other_sites_ms_per_step'].items()})"
done; done
