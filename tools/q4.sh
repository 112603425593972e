#!/bin/bash
export PYTHONUNBUFFERED=1
timeout -s KILL 900 python -m pytest tests/test_gpu_gemm.py tests/test_gpu_parity.py -x -q > gpurun_out/q4_tests.log 2>&1; echo "tests rc=$?"; tail -1 gpurun_out/q4_tests.log
for i in 1 2; do
timeout -s KILL 600 python bench.py --steps 20 --cpu-sample-outputs 16 > gpurun_out/q4.log 2>&1
python - <<PY
import json
d=json.loads(open('gpurun_out/q4.log').read().strip().splitlines()[-1])
print('ms/step', round(d['ms_per_step'],4), {k: round(v,3) for k,v in d['roofline']['other_sites_ms_per_step'].items()})
PY
done
bash tools/prof_full.sh tcrow2 "k_tc_row" 5 > /dev/null 2>&1; python tools/ncu_table.py gpurun_out/full_tcrow2_raw.csv 2>&1 | head -7; rm -f gpurun_out/full_tcrow2.ncu-rep gpurun_out/full_tcrow2_source.csv
