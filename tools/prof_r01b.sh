#!/bin/bash
# One bench step (tools/prof_step.py) under ncu: the launch list and a --set full capture of every kernel.
# Reports are reduced to CSV on the box (gpurun_out/ is capped at 64 MiB).
export PYTHONUNBUFFERED=1
TAG=${1:-r01b}
REGEX=${2:-.}
timeout -s KILL 600 ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/launches_${TAG}.csv python tools/prof_step.py > gpurun_out/launches_${TAG}.log 2>&1; echo "launches rc=$?"
timeout -s KILL 1500 ncu --profile-from-start off --set full --clock-control none --import-source on -k regex:"$REGEX" \
  -o /tmp/full_${TAG} python tools/prof_step.py > gpurun_out/full_${TAG}.log 2>&1; echo "full rc=$?"
ncu -i /tmp/full_${TAG}.ncu-rep --page raw --csv > gpurun_out/full_${TAG}_raw.csv 2>/dev/null
ncu -i /tmp/full_${TAG}.ncu-rep --page details --csv > gpurun_out/full_${TAG}_details.csv 2>/dev/null
ls -la /tmp/full_${TAG}.ncu-rep
if [ $(stat -c %s /tmp/full_${TAG}.ncu-rep) -lt 40000000 ]; then cp /tmp/full_${TAG}.ncu-rep gpurun_out/; fi
