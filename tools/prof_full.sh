#!/bin/bash
# --set full capture of the kernels matching $2 in one step; reduces to raw/details CSV on the box.
export PYTHONUNBUFFERED=1
TAG=$1; REGEX=$2; COUNT=${3:-8}
timeout -s KILL 1200 ncu --profile-from-start off --set full --clock-control none --import-source on -k regex:"$REGEX" -c $COUNT \
  -o /tmp/full_${TAG} python tools/prof_step.py > gpurun_out/full_${TAG}.log 2>&1; echo "ncu $TAG rc=$?"
ncu -i /tmp/full_${TAG}.ncu-rep --page raw --csv > gpurun_out/full_${TAG}_raw.csv 2>/dev/null
ncu -i /tmp/full_${TAG}.ncu-rep --page details --csv > gpurun_out/full_${TAG}_details.csv 2>/dev/null
ncu -i /tmp/full_${TAG}.ncu-rep --page source --csv -k regex:"$REGEX" > gpurun_out/full_${TAG}_source.csv 2>/dev/null
ls -la /tmp/full_${TAG}.ncu-rep
if [ $(stat -c %s /tmp/full_${TAG}.ncu-rep) -lt 30000000 ]; then cp /tmp/full_${TAG}.ncu-rep gpurun_out/; fi
