# quick GPU correctness pass: selected test files (args) with per-test timeout
OUT=gpurun_out
timeout 1200 python -m pytest "$@" -m gpu -q --timeout 180 --maxfail=40 -p no:cacheprovider > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?"
grep -E "passed|failed|FAILED|Error" $OUT/pytest_gpu.log | tail -30
