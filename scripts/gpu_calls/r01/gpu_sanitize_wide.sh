# compute-sanitizer on the wide (256x512) pair kernel (forced with SVP_TC_WIDE=2) and the fixed hist256 / FFMA release
OUT=gpurun_out
for tool in memcheck racecheck synccheck; do
  SVP_TC_WIDE=2 timeout 900 compute-sanitizer --tool $tool --error-exitcode 99 --target-processes all python -m pytest tests/test_gpu_sgemm_tc.py tests/test_gpu_parity.py -m gpu -q -p no:cacheprovider -k "(ragged_alpha_beta and device and sgemm-2) or (mixed_small and device and coalesced_interleaved) or sgemm_alpha_beta" > $OUT/sanitize_wide_$tool.log 2>&1; echo "$tool rc=$?"
  grep -E "ERROR SUMMARY|passed|failed|Hazard|hazard" $OUT/sanitize_wide_$tool.log | sort | uniq -c | tail -6
done
