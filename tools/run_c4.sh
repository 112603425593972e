export PYTHONUNBUFFERED=1
timeout -s KILL 300 python -m pytest tests/test_gpu_gemm.py tests/test_gpu_parity.py -x -q > gpurun_out/tests_c4c.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/tests_c4c.log
timeout -s KILL 600 python bench.py --config C4 --steps 3 --warmup 3 > gpurun_out/bench_c4c.log 2>&1; echo c4 rc=$?
python -c "
import json; d=json.loads(open('gpurun_out/bench_c4c.log').read().strip().splitlines()[-1]); print('C4 ms', d['ms_per_step'], 'K', d['config']['K'])"
bash tools/launches.sh c4c --config C4 --K 2 --group 1 | head -12
