#!/bin/bash
# C5 (papers100M-shaped) bench, guarded by the box's host memory (run under gpurun).
export PYTHONUNBUFFERED=1
free -g; nproc; nvidia-smi --query-gpu=memory.total,memory.used --format=csv
MEM=$(free -g | awk '/Mem:/ {print $7}')
: skip scaled
if [ "$MEM" -lt 90 ]; then echo "host memory $MEM GB < 90: skipping full C5"; exit 0; fi
( while true; do free -g | awk '/Mem:/ {print "host used", $3}' >> gpurun_out/c5_mem.log; nvidia-smi --query-gpu=memory.used --format=csv,noheader >> gpurun_out/c5_mem.log; sleep 10; done ) &
MON=$!
timeout -s KILL 1200 python bench.py --config C5 --steps 5 --warmup 3 ${C5_ARGS} > gpurun_out/c5.log 2> gpurun_out/c5.err; echo "c5 rc=$?"
kill $MON
tail -c 3000 gpurun_out/c5.log; tail -40 gpurun_out/c5.err
