python -m pytest tests -m gpu -x -q 2>&1 | tail -2
for v in "" "BETTY_AGG_NOHINT=1" "BETTY_AGG_NOORDER=1" "BETTY_AGG_NOHINT=1 BETTY_AGG_NOORDER=1"; do
  env $v python bench.py --steps 10 > gpurun_out/b.log 2>&1
  python -c "
import json; d=json.loads(open('gpurun_out/b.log').read().strip().splitlines()[-1]); print('$v', 'ms/step', round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['roofline']['other_sites_ms_per_step'].items()})"
done
