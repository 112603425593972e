#!/bin/bash
# compute-sanitizer over the small GPU cases (run under gpurun): memcheck, racecheck and synccheck on
# smoke() (REG, fp32 and bf16 fused steps: extraction, gather4 pipeline, tcgen05 / 3xTF32 GEMMs,
# loss, backward, Adam) and on a few parity / GEMM tests.  Summaries -> gpurun_out/sanitize_<tool>.txt
export PYTHONUNBUFFERED=1
OUT=gpurun_out
SMOKE='python -c "import __graft_entry__ as g; g.smoke()"'
TESTS='python -m pytest -q -x -p no:cacheprovider tests/test_gpu_gemm.py -k "300-209-256 or 127-64-48" tests/test_gpu_parity.py -k "golden or mean2-fp32 or mean2-bf16 or pool2-fp32 or hub_rows"'
for tool in memcheck racecheck synccheck; do
  {
    echo "== compute-sanitizer --tool $tool: smoke()"
    timeout -s KILL 1200 compute-sanitizer --tool $tool --print-limit 20 bash -c "$SMOKE" 2>&1 | tail -25
    echo "== compute-sanitizer --tool $tool: selected tests"
    timeout -s KILL 1500 compute-sanitizer --tool $tool --print-limit 20 bash -c "$TESTS" 2>&1 | tail -25
  } > $OUT/sanitize_$tool.txt
  echo "$tool: $(grep -c 'ERROR SUMMARY: 0 errors' $OUT/sanitize_$tool.txt) clean summaries"
done
