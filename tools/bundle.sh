#!/bin/bash
# Full round bundle in one gpurun call: GPU tests + smoke, bench lines C1-C5 + the reference arm,
# C3 launch lists (cold / warm, bf16 and fp32), ncu --set full of the top C3 kernels, per-rank shares.
# Outputs gpurun_out/*_${TAG}*; copy the ones to keep into profiles/.
export PYTHONUNBUFFERED=1
TAG=${1:-r06}
timeout -s KILL 1500 python -m pytest tests -m gpu -x -q > gpurun_out/tests_${TAG}.log 2>&1; echo "tests rc=$?"; tail -1 gpurun_out/tests_${TAG}.log
python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" 2>&1 | tail -1
for C in C3 C1 C2 C4 C5; do
  timeout -s KILL 1200 python bench.py --config $C > gpurun_out/bench_${C}_${TAG}.log 2>&1; echo "$C bench rc=$?"
  tail -1 gpurun_out/bench_${C}_${TAG}.log > gpurun_out/bench_${C}_${TAG}.jsonl
done
timeout -s KILL 900 python bench.py --impl reference > gpurun_out/bench_reference_${TAG}.log 2>&1; echo "reference rc=$?"
tail -1 gpurun_out/bench_reference_${TAG}.log > gpurun_out/bench_reference_${TAG}.jsonl
bash tools/launches.sh C3_${TAG} > gpurun_out/launches_C3_${TAG}.txt 2>&1
CACHE=none bash tools/launches.sh C3w_${TAG} > gpurun_out/launches_C3_warm_${TAG}.txt 2>&1
CACHE=none bash tools/launches.sh fp32w_${TAG} --mode fp32 > gpurun_out/launches_fp32_warm_${TAG}.txt 2>&1
CACHE=none bash tools/launches.sh freshw_${TAG} --fresh > gpurun_out/launches_fresh_warm_${TAG}.txt 2>&1
bash tools/prof_full.sh ${TAG} "k_agg_mean|k_tc_row|k_tc_red|k_relabel|k_mark_new|k_csc_pf_v" 12 > /dev/null 2>&1; echo "full rc=$?"
python tools/ncu_table.py gpurun_out/full_${TAG}_raw.csv > gpurun_out/ncu_${TAG}.txt 2>&1
python tools/ncu_src.py gpurun_out/full_${TAG}_source.csv k_agg_mean 25 >> gpurun_out/ncu_${TAG}.txt 2>&1
rm -f gpurun_out/full_${TAG}.ncu-rep gpurun_out/full_${TAG}_details.csv
bash tools/sim_world.sh > gpurun_out/sim_world_${TAG}.txt 2>&1
for f in gpurun_out/bench_*_${TAG}.jsonl; do
python - "$f" <<'PY'
import json, sys
f = sys.argv[1]
try:
    d = json.loads(open(f).read())
    r = d.get('roofline') or {}
    e = d.get('e2e') or {}
    pp = (d.get('paper_precision') or {}).get('ms_per_step')
    print(f, 'ms/step', round(d['ms_per_step'], 3), 'G/s', round(d['value'] / 1e9, 3), 'frac', r.get('frac'),
          'e2e ms', e.get('ms_per_step'), 'fp32 ms', pp, 'clocks', d.get('clocks'))
except Exception as ex:
    print(f, 'unreadable', ex)
PY
done
