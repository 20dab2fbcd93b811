# SGEMM tail split: parity tests, wave probe, bench A/B (SVP_SGEMM_TAIL=0/1 alternating)
OUT=gpurun_out
timeout 1200 python -m pytest tests/test_gpu_sgemm_tc.py tests/test_gpu_parity.py -q --timeout 600 -p no:cacheprovider -k "tail_split or config5 or 2048_sampled or ragged_alpha_beta or config2" > $OUT/pytest_tail.log 2>&1; echo "pytest rc=$?"; tail -3 $OUT/pytest_tail.log
timeout 600 python tools/sgemm_waves.py 48 50 51 52 > $OUT/sgemm_waves_tail.log 2>&1; cat $OUT/sgemm_waves_tail.log
for r in 1 2; do for t in 0 1; do
  SVP_SGEMM_TAIL=$t timeout 900 python bench.py --no-serial --no-alt --no-e2e --no-cpu > $OUT/bench_tail${t}_$r.log 2>&1
done; done
