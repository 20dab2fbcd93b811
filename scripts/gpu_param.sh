OUT=gpurun_out
timeout 900 python -m pytest tests/test_gpu_f4.py tests/test_gpu_parity.py -m gpu -q --timeout 300 -p no:cacheprovider > $OUT/pytest_param.log 2>&1; echo "pytest rc=$?"; tail -2 $OUT/pytest_param.log; grep -E "^FAILED|Error" $OUT/pytest_param.log | head
for tm in 1 0; do
  timeout 300 python bench.py --steps 30 --warmup 3 --no-e2e --no-cpu --no-serial --no-alt --table-mode $tm > $OUT/bench_tm$tm.log 2>&1; echo "bench tm=$tm rc=$?"
done
timeout 600 python tools/sweeps.py --only 6 --out $OUT/sweeps_f4b.json > /dev/null 2>&1; echo "sweep rc=$?"
