# TF32+2xBF16 sgemm: parity first, then A/B bench vs 3xTF32
OUT=gpurun_out
mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_sgemm_tc.py -m gpu -q --timeout 300 -p no:cacheprovider -x > $OUT/pytest_tc.log 2>&1; echo "pytest tc rc=$?"; grep -E "passed|failed|FAILED|Error|assert" $OUT/pytest_tc.log | head -20
for impl in tf32bf16 3xtf32; do
  timeout 600 python bench.py --steps 30 --warmup 3 --no-e2e --no-cpu --no-serial --sgemm-impl $impl --alt-impl $( [ $impl = 3xtf32 ] && echo tf32bf16 || echo 3xtf32 ) > $OUT/bench_$impl.log 2>&1; echo "bench $impl rc=$?"
done
