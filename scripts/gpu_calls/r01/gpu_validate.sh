# validate_ptrs range cache (1) vs per-submit queries (2); 64-segment param cap; GPU tests
OUT=gpurun_out
timeout 1500 python -m pytest tests -m gpu -q --timeout 300 -p no:cacheprovider > $OUT/pytest_gpu_val.log 2>&1; echo "pytest rc=$?"; tail -2 $OUT/pytest_gpu_val.log
timeout 600 python tools/s1_probe.py > $OUT/s1_probe_val.jsonl 2>&1; echo "s1 rc=$?"
for r in 1 2; do for v in 1 2; do
  SVP_SWEEP_VALIDATE=$v timeout 900 python tools/sweeps.py --only 6 --out $OUT/sweeps_s6_val${v}_$r.json > /dev/null 2>&1
done; done
timeout 900 python bench.py --no-serial --no-alt --no-e2e --no-cpu > $OUT/bench_val.log 2>&1; echo "bench rc=$?"
