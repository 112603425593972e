#!/bin/bash
# agg_l0 experiment: column passes (working-set budget) with CTA-level dynamic claiming
python -m pytest tests -m gpu -x -q 2>&1 | tail -1
for v in 1000000 60 40 25; do
  BETTY_AGG_WS_MB=$v python bench.py --steps 10 > gpurun_out/b.log 2>&1
  python -c "
import json; d=json.loads(open('gpurun_out/b.log').read().strip().splitlines()[-1]); print('WS $v', 'ms/step', round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['roofline']['other_sites_ms_per_step'].items()})"
  BETTY_AGG_WS_MB=$v timeout 600 ncu --profile-from-start off --metrics gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:"k_agg_mean_xa" --csv --log-file gpurun_out/agg_$v.csv python tools/prof_step.py > /dev/null 2>&1
  python - <<PY
import csv
rows=list(csv.reader(open('gpurun_out/agg_$v.csv')))
hi=next(i for i,r in enumerate(rows) if 'Kernel Name' in r); h=rows[hi]
iid,im,iv=h.index('ID'),h.index('Metric Name'),h.index('Metric Value')
out={}
for r in rows[hi+1:]:
    if len(r)>iv: out.setdefault(r[iid],{})[r[im]]=r[iv]
for k,d in out.items(): print('   launch', k, d)
PY
done
