#!/bin/bash
# --set full capture (with source) of the kernels matching $2 in one step; keeps the .ncu-rep if small
export PYTHONUNBUFFERED=1
TAG=$1; REGEX=$2
timeout -s KILL 900 ncu --profile-from-start off --set full --clock-control none --import-source on -k regex:"$REGEX" \
  -o gpurun_out/k_${TAG} python tools/prof_step.py > gpurun_out/k_${TAG}.log 2>&1; echo "ncu $TAG rc=$?"
ncu -i gpurun_out/k_${TAG}.ncu-rep --page raw --csv > gpurun_out/k_${TAG}_raw.csv 2>/dev/null
ls -la gpurun_out/k_${TAG}.ncu-rep
