#!/bin/bash
# C3: epoch time vs micro-batch count K and vs partition (the paper's Table 6 / Fig. 16 analogues)
export PYTHONUNBUFFERED=1
for K in 8 16 32 64; do for P in reg random range; do
  timeout -s KILL 600 python bench.py --K $K --partition $P --steps 10 --cpu-sample-outputs 16 > gpurun_out/sw.log 2>&1
  python - <<PY
import json
d=json.loads(open('gpurun_out/sw.log').read().strip().splitlines()[-1])
p=d['plan']
print(f"K={$K:3d} part=$P  ms/step={d['ms_per_step']:.3f}  Gedges/s={d['value']/1e9:.2f}  edges/step={d['edges_per_step']/1e6:.2f}M  layer0 n_src={p['n_src'][0]/1e6:.2f}M  layer0 E={p['edges'][0]/1e6:.2f}M  full-batch E={d['full_batch_edges']/1e6:.2f}M")
PY
done; done
