#!/bin/bash
# Round profile bundle (run under gpurun): bench line, launch list of one step, ncu --set full of the
# dominant kernels; reduced to CSV/text under gpurun_out/ (copy to profiles/ afterwards).
export PYTHONUNBUFFERED=1
TAG=${1:-r01d}
timeout -s KILL 900 python bench.py > gpurun_out/bench_${TAG}.log 2>&1; echo "bench rc=$?"
tail -1 gpurun_out/bench_${TAG}.log > gpurun_out/bench_${TAG}.jsonl
bash tools/launches.sh ${TAG} > gpurun_out/launches_${TAG}.txt 2>&1; echo "launches rc=$?"
bash tools/prof_full.sh ${TAG} "k_agg_mean|k_tc_row|k_tc_red|k_relabel|k_mark_new|k_csc_pf_v" 12 > /dev/null 2>&1; echo "full rc=$?"
python tools/ncu_table.py gpurun_out/full_${TAG}_raw.csv > gpurun_out/ncu_${TAG}.txt 2>&1
python tools/ncu_src.py gpurun_out/full_${TAG}_source.csv k_agg_mean 25 >> gpurun_out/ncu_${TAG}.txt 2>&1
rm -f gpurun_out/full_${TAG}.ncu-rep
