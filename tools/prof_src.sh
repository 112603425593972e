#!/bin/bash
# --set full + source capture of the kernels matching $2 in one step; exports raw metrics and
# per-kernel SASS source tables (stall samples) as CSV, drops the report (gpurun_out/ cap)
export PYTHONUNBUFFERED=1
TAG=$1; REGEX=$2
timeout -s KILL 1200 ncu --profile-from-start off --set full --clock-control none --import-source on -k regex:"$REGEX" \
  -o /tmp/k_${TAG} python tools/prof_step.py > gpurun_out/k_${TAG}.log 2>&1; echo "ncu $TAG rc=$?"
ncu -i /tmp/k_${TAG}.ncu-rep --page raw --csv > gpurun_out/k_${TAG}_raw.csv 2>/dev/null
ncu -i /tmp/k_${TAG}.ncu-rep --page source --csv --print-source sass 2>/dev/null | gzip > gpurun_out/k_${TAG}_src.csv.gz
ls -la /tmp/k_${TAG}.ncu-rep gpurun_out/k_${TAG}_src.csv.gz
