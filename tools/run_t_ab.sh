export PYTHONUNBUFFERED=1
timeout -s KILL 600 python -m pytest tests -m gpu -x -q > gpurun_out/tests_g4e.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/tests_g4e.log
bash tools/ab_agg.sh ab3
