# profile_level 2 (measured per-VP split): GPU tests, default bench (no-regression check)
OUT=gpurun_out
timeout 1500 python -m pytest tests -m gpu -q --timeout 300 -p no:cacheprovider > $OUT/pytest_gpu_prof2.log 2>&1; echo "pytest rc=$?"; tail -3 $OUT/pytest_gpu_prof2.log
timeout 1200 python bench.py > $OUT/bench_prof2.log 2>&1; echo "bench rc=$?"
