export PYTHONUNBUFFERED=1
timeout -s KILL 600 python -m pytest tests -m gpu -x -q > gpurun_out/tests_pool8.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/tests_pool8.log
for A in 0 1; do
BETTY_POOL_ARG32=$A timeout -s KILL 600 python bench.py --config C4 --steps 3 --warmup 3 > gpurun_out/bench_c4_$A.log 2>&1; echo c4 rc=$?
python -c "
import json; d=json.loads(open('gpurun_out/bench_c4_$A.log').read().strip().splitlines()[-1]); print('C4 arg32=$A ms', d['ms_per_step'], 'K', d['config']['K'])"
done
bash tools/launches.sh c4d --config C4 --K 2 --group 1 | head -8
