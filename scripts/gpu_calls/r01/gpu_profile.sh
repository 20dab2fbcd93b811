# GPU check + profiling pass: tests, smoke, bench, ncu launch list, ncu full captures.
set -x
OUT=gpurun_out
timeout 1500 python -m pytest tests -m gpu -q --timeout 300 --maxfail=30 -p no:cacheprovider > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?"
tail -5 $OUT/pytest_gpu.log
timeout 900 python bench.py --steps 30 --warmup 3 > $OUT/bench.log 2>&1; echo "bench rc=$?"
tail -2 $OUT/bench.log
BENCH_SMALL="python bench.py --steps 2 --warmup 3 --no-serial --no-e2e --no-cpu"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:k_ --csv --log-file $OUT/launches.csv $BENCH_SMALL > $OUT/ncu_launches.log 2>&1; echo "ncu list rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_sgemm_ffma -s 1 -c 1 -o $OUT/prof_sgemm -f $BENCH_SMALL > $OUT/ncu_sgemm.log 2>&1; echo "ncu sgemm rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_vecadd|k_saxpy|k_hist256|k_blackscholes" -s 4 -c 4 -o $OUT/prof_mem -f $BENCH_SMALL > $OUT/ncu_mem.log 2>&1; echo "ncu mem rc=$?"
ls -la $OUT
