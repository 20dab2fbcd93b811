OUT=gpurun_out
timeout 300 python -m pytest tests/test_gpu_sgemm_tc.py -m gpu -q --timeout 120 -p no:cacheprovider -x > $OUT/pytest_st.log 2>&1; echo "pytest rc=$?"; tail -1 $OUT/pytest_st.log
timeout 600 python scripts/sgemm_accuracy.py > $OUT/sgemm_accuracy.json 2> $OUT/sgemm_accuracy.err; echo "acc rc=$?"
for r in 1 2; do for impl in tf32bf16 3xtf32; do
  timeout 300 python bench.py --steps 30 --warmup 3 --no-e2e --no-cpu --no-serial --no-alt --sgemm-impl $impl > $OUT/bench_st7_${impl}_$r.log 2>&1; echo "bench $impl $r rc=$?"
done; done
