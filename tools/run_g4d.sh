export PYTHONUNBUFFERED=1
timeout -s KILL 600 python -m pytest tests -m gpu -x -q > gpurun_out/tests_g4d.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/tests_g4d.log
bash tools/ab_agg.sh ab2
timeout -s KILL 600 python bench.py --config C4 --steps 3 --warmup 3 > gpurun_out/bench_c4b.log 2>&1; echo c4 rc=$?
python -c "
import json; d=json.loads(open('gpurun_out/bench_c4b.log').read().strip().splitlines()[-1]); print('C4 ms', d['ms_per_step'], 'K', d['config']['K'])"
bash tools/launches.sh c4b --config C4 --K 2 --group 1 | head -12
