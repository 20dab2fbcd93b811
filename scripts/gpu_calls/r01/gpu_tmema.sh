# SPLIT 4 (A-side bf16 in TMEM): parity (pair and single CTA), then A/B bench
OUT=gpurun_out
for pair in 1 0; do
  SVP_TC_CTA_PAIR=$pair timeout 300 python -m pytest tests/test_gpu_sgemm_tc.py -m gpu -q --timeout 120 -p no:cacheprovider -x > $OUT/pytest_ta_$pair.log 2>&1; rc=$?; echo "pytest pair=$pair rc=$rc"; tail -1 $OUT/pytest_ta_$pair.log
  [ $rc -ne 0 ] && grep -E "assert|Error" $OUT/pytest_ta_$pair.log | head -5 && exit 0
done
for r in 1 2; do for ta in 1 0; do
  SVP_TC_TMEM_A=$ta timeout 300 python bench.py --steps 30 --warmup 3 --no-e2e --no-cpu --no-serial --no-alt > $OUT/bench_ta${ta}_$r.log 2>&1; echo "bench ta=$ta rc=$?"
done; done
