# re-entry verification: GPU tests, smoke, default bench, reference arm
OUT=gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.limit --format=csv > $OUT/gpu_info.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q --timeout 300 -p no:cacheprovider > $OUT/pytest_gpu_full.log 2>&1; echo "pytest rc=$?"; tail -2 $OUT/pytest_gpu_full.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?"
timeout 1200 python bench.py > $OUT/bench_full.log 2>&1; echo "bench rc=$?"; tail -1 $OUT/bench_full.log | cut -c1-600
