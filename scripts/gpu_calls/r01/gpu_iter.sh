# iteration loop: correctness of the touched kernels, bench (3xtf32), ncu of the top kernels
OUT=gpurun_out
timeout 900 python -m pytest tests/test_gpu_sgemm_tc.py tests/test_gpu_parity.py -m gpu -q --timeout 180 -p no:cacheprovider > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?"; grep -E "passed|failed|FAILED" $OUT/pytest_gpu.log | tail -8
timeout 900 python bench.py --steps 30 --warmup 3 --sgemm-impl 3xtf32 --no-cpu --no-e2e > $OUT/bench_3xtf32.log 2>&1; echo "bench rc=$?"
BENCH_SMALL="python bench.py --steps 2 --warmup 3 --no-serial --no-e2e --no-cpu --sgemm-impl 3xtf32"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_sgemm_tc|k_hist256" -s 2 -c 2 -o $OUT/prof_iter -f $BENCH_SMALL > $OUT/ncu_iter.log 2>&1; echo "ncu rc=$?"
