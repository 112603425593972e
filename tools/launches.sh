#!/bin/bash
# launch list (per-kernel time + DRAM bytes) of one step: bash tools/launches.sh TAG [prof_step args...]
export PYTHONUNBUFFERED=1
TAG=$1; shift
# CACHE=none: warm caches (ncu's default flushes them before every kernel)
timeout -s KILL 900 ncu --profile-from-start off --cache-control ${CACHE:-all} --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
  --log-file gpurun_out/launches_${TAG}.csv python tools/prof_step.py "$@" > gpurun_out/launches_${TAG}.log 2>&1; echo "launches rc=$?"
python tools/launch_summary.py gpurun_out/launches_${TAG}.csv | head -40
