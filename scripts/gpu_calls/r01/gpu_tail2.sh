# SGEMM tail split only when alone: tests, bench x2, one-stream cfg5 soak (tail + dynamic order)
OUT=gpurun_out
timeout 1500 python -m pytest tests -m gpu -q --timeout 600 -p no:cacheprovider > $OUT/pytest_tail2.log 2>&1; echo "pytest rc=$?"; tail -2 $OUT/pytest_tail2.log
for r in 1 2; do timeout 900 python bench.py > $OUT/bench_tail2_$r.log 2>&1; done
timeout 900 python scripts/cfg5_soak.py 4 0:0:1:0 0:1:1:0 > $OUT/soak_tail.log 2>&1; grep combo $OUT/soak_tail.log
