#!/bin/bash
# L2 reuse of the layer-0 gather vs graph scale (feature table 0.51 GB at scale 1)
python -m pytest tests -m gpu -x -q 2>&1 | tail -1
for sc in 0.05 0.1 0.2 0.35 0.5 1.0; do
  timeout 600 ncu --profile-from-start off --metrics gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:"k_agg_mean_xa|k_relabel" --csv --log-file gpurun_out/l2_$sc.csv python tools/prof_step.py --scale $sc > gpurun_out/l2_$sc.log 2>&1
done
python - <<'PY'
import csv
for sc in ['0.05','0.1','0.2','0.35','0.5','1.0']:
    rows=list(csv.reader(open(f'gpurun_out/l2_{sc}.csv')))
    hi=next(i for i,r in enumerate(rows) if 'Kernel Name' in r); h=rows[hi]
    ik,im,iv=h.index('Kernel Name'),h.index('Metric Name'),h.index('Metric Value')
    out={}
    for r in rows[hi+1:]:
        if len(r)>iv: out.setdefault(r[ik][:22],{})[r[im]]=r[iv]
    print(sc, open(f'gpurun_out/l2_{sc}.log').read().strip().splitlines()[-1][:90])
    for k,v in out.items(): print('   ',k,v)
PY
