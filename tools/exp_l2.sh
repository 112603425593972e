#!/bin/bash
# L2 reuse of the layer-0 gather vs graph scale (feature table 0.51 GB at scale 1)
for sc in 0.05 0.1 0.2 0.35 0.5 1.0; do
  echo "== scale $sc"
  timeout 600 ncu --profile-from-start off --metrics gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:"k_agg_mean_xa" --csv python tools/prof_step.py --scale $sc 2>/dev/null | grep -E "k_agg|prof_step" | awk -F'","' '{print $(NF-2), $NF}'
  python tools/prof_step.py --scale $sc 2>/dev/null | grep prof_step
done
