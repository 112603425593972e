#!/bin/bash
# launch-group size: all 32 micro-batches vs groups of 16 / 8
for g in 0 16 8; do
  python bench.py --steps 10 --group $g > gpurun_out/b.log 2>&1
  python -c "
import json; d=json.loads(open('gpurun_out/b.log').read().strip().splitlines()[-1]); print('group $g', 'ms/step', round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['roofline']['other_sites_ms_per_step'].items()}, d['plan']['kernels_per_step'])"
done
