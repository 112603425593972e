#!/bin/bash
# Final round check + bundle: full GPU tests, smoke, C3/C4/C5 bench lines, C3 launch list, ncu of top kernels
export PYTHONUNBUFFERED=1
TAG=${1:-r01h}
timeout -s KILL 1200 python -m pytest tests -m gpu -x -q > gpurun_out/tests_${TAG}.log 2>&1; echo "tests rc=$?"; tail -1 gpurun_out/tests_${TAG}.log
python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" 2>&1 | tail -1
bash tools/prof_bundle.sh ${TAG}
