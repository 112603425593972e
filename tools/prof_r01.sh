#!/bin/bash
# ncu --set full captures of the hot kernels of one bench step (run under gpurun).
export PYTHONUNBUFFERED=1
A="--steps 1 --warmup 1 --e2e-steps 1 --cpu-sample-outputs 16"
TAG=${1:-r01}
run() { timeout -s KILL 900 ncu --set full --clock-control none --import-source on -k regex:"$1" -s $2 -c $3 -o gpurun_out/prof_${TAG}_$4 python bench.py $A > gpurun_out/ncu_${TAG}_$4.log 2>&1; echo "$4 rc=$?"; }
run "k_agg_mean_xa" 1 1 agg
run "k_tc_row" 3 3 tcrow
run "k_relabel|k_mark_new" 132 4 extract
run "k_segsort_warp|k_reg_rows_warp|k_tc_red|k_csc_pf" 6 6 misc
