#!/bin/bash
# Round profile bundle (run under gpurun): C3 bench line, launch list, ncu --set full of the top kernels,
# C4 / C5 bench lines, C5 launch list.  Copy gpurun_out/*_${TAG}* to profiles/ afterwards.
export PYTHONUNBUFFERED=1
TAG=${1:-r01g}
timeout -s KILL 900 python bench.py > gpurun_out/bench_C3_${TAG}.log 2>&1; echo "C3 bench rc=$?"
tail -1 gpurun_out/bench_C3_${TAG}.log > gpurun_out/bench_C3_${TAG}.jsonl
bash tools/launches.sh C3_${TAG} > gpurun_out/launches_C3_${TAG}.txt 2>&1; echo "launches rc=$?"
bash tools/prof_full.sh ${TAG} "k_agg_mean|k_tc_row|k_tc_red|k_relabel|k_mark_new|k_csc_pf_v" 12 > /dev/null 2>&1; echo "full rc=$?"
python tools/ncu_table.py gpurun_out/full_${TAG}_raw.csv > gpurun_out/ncu_${TAG}.txt 2>&1
python tools/ncu_src.py gpurun_out/full_${TAG}_source.csv k_agg_mean 25 >> gpurun_out/ncu_${TAG}.txt 2>&1
python tools/traffic.py gpurun_out/full_${TAG}_raw.csv k_agg_mean C3:K32:bf16:n1 agg_l0
rm -f gpurun_out/full_${TAG}.ncu-rep gpurun_out/full_${TAG}_details.csv
timeout -s KILL 900 python bench.py --config C4 --steps 5 > gpurun_out/bench_C4_${TAG}.log 2>&1; echo "C4 bench rc=$?"
tail -1 gpurun_out/bench_C4_${TAG}.log > gpurun_out/bench_C4_${TAG}.jsonl
timeout -s KILL 1200 python bench.py --config C5 --steps 5 > gpurun_out/bench_C5_${TAG}.log 2>&1; echo "C5 bench rc=$?"
tail -1 gpurun_out/bench_C5_${TAG}.log > gpurun_out/bench_C5_${TAG}.jsonl
bash tools/launches.sh C5_${TAG} --config C5 --K 32 --group 12 > gpurun_out/launches_C5_${TAG}.txt 2>&1; echo "C5 launches rc=$?"
for f in gpurun_out/bench_C3_${TAG}.jsonl gpurun_out/bench_C4_${TAG}.jsonl gpurun_out/bench_C5_${TAG}.jsonl; do
python - <<PY
import json
d=json.loads(open('$f').read())
r=d.get('roofline') or {}
print('$f', 'ms/step', round(d['ms_per_step'],3), 'Gedges/s', round(d['value']/1e9,3), 'frac', r.get('frac'), 'e2e', round(d['e2e']['value']/1e9,3))
PY
done
