# CTA-pair (cta_group::2) tcgen05 SGEMM: parity first (short timeouts), then A/B bench
OUT=gpurun_out
mkdir -p $OUT
timeout 300 python -m pytest tests/test_gpu_sgemm_tc.py -m gpu -q --timeout 120 -p no:cacheprovider -x > $OUT/pytest_pair.log 2>&1; rc=$?; echo "pytest pair rc=$rc"; grep -E "passed|failed|FAILED|Error|assert|Timeout" $OUT/pytest_pair.log | head -20
if [ $rc -ne 0 ]; then exit 0; fi
for impl in tf32bf16 3xtf32; do
  for pair in 1 0; do
    SVP_TC_CTA_PAIR=$pair timeout 300 python bench.py --steps 30 --warmup 3 --no-e2e --no-cpu --no-serial --no-alt --sgemm-impl $impl > $OUT/bench_${impl}_pair$pair.log 2>&1; echo "bench $impl pair=$pair rc=$?"
  done
done
