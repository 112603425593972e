#!/bin/bash
# C4: memory-aware micro-batch count under several capacities (the paper's Table 2 / Fig. 10 analogue)
export PYTHONUNBUFFERED=1
for CAP in 48 24 16 12; do
  timeout -s KILL 900 python bench.py --config C4 --capacity-gb $CAP --steps 3 --warmup 3 --cpu-sample-outputs 1 > gpurun_out/swm.log 2>&1
  python - <<PY
import json
d=json.loads(open('gpurun_out/swm.log').read().strip().splitlines()[-1])
m=d['memory_aware']; p=d['plan']
print(f"capacity={$CAP:3d} GB  K={m['K']:3d}  peak estimate={m['peak_estimate_gb']:.2f} GB  search={m['search_s']:.2f} s  ms/step={d['ms_per_step']:.1f}  edges/step={d['edges_per_step']/1e6:.1f}M  plan arena={p['arena_bytes']/2**30:.1f} GB")
PY
done
