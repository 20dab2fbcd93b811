OUT=gpurun_out
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 99 --target-processes all python -m pytest tests/test_gpu_parity.py -m gpu -q -p no:cacheprovider -k "mixed_small and device and coalesced_interleaved or sgemm_alpha_beta" > $OUT/sanitize_$tool.log 2>&1; echo "$tool rc=$?"
  grep -E "ERROR SUMMARY|passed|failed" $OUT/sanitize_$tool.log | tail -3
done
timeout 900 compute-sanitizer --tool memcheck --error-exitcode 99 python -m pytest tests/test_gpu_sgemm_tc.py -m gpu -q -p no:cacheprovider -k "ragged and device" > $OUT/sanitize_tc.log 2>&1; echo "memcheck tc rc=$?"; grep -E "ERROR SUMMARY|passed|failed" $OUT/sanitize_tc.log | tail -3
