#!/bin/bash
# agg_l0 experiment: column passes (working-set budget) and order switches
python -m pytest tests -m gpu -x -q 2>&1 | tail -2
for v in "BETTY_AGG_WS_MB=1000000" "BETTY_AGG_WS_MB=40" "BETTY_AGG_NOORDER=1"; do
  env $v python bench.py --steps 10 > gpurun_out/b.log 2>&1
  python -c "
import json; d=json.loads(open('gpurun_out/b.log').read().strip().splitlines()[-1]); print('$v', 'ms/step', round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['roofline']['other_sites_ms_per_step'].items()})"
done
for v in 1000000 40; do
BETTY_AGG_WS_MB=$v timeout 600 ncu --profile-from-start off --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:"k_agg_mean_xa|k_csc|k_reg_rows" --csv python tools/prof_step.py 2>/dev/null | grep -E "k_agg|k_csc|k_reg" | awk -F'","' '{print substr($5,1,40), $(NF-2), $NF}'
done
