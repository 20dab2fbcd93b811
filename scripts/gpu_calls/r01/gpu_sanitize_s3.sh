# compute-sanitizer on the session-3 paths: hist ragged staging (+ single-launch form),
# dynamic tile order, profile_level 2 busy counters, sized param tables
OUT=gpurun_out
SEL="hist256_ragged or dynamic_tile_order or measured_split or (mixed_small and device and coalesced_interleaved)"
for tool in memcheck racecheck synccheck; do
  timeout 1200 compute-sanitizer --tool $tool --error-exitcode 99 --target-processes all python -m pytest tests/test_gpu_parity.py -m gpu -q -p no:cacheprovider -k "$SEL" > $OUT/san3_$tool.log 2>&1; echo "$tool rc=$?"
  grep -E "ERROR SUMMARY|RACECHECK SUMMARY|passed|failed" $OUT/san3_$tool.log | tail -3
done
for tool in memcheck racecheck; do
  SVP_HIST_FUSED=1 timeout 900 compute-sanitizer --tool $tool --error-exitcode 99 python -m pytest tests/test_gpu_parity.py -m gpu -q -p no:cacheprovider -k "hist256_ragged" > $OUT/san3_fused_$tool.log 2>&1; echo "fused $tool rc=$?"
  grep -E "ERROR SUMMARY|RACECHECK SUMMARY|passed|failed" $OUT/san3_fused_$tool.log | tail -3
done
