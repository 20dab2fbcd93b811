OUT=gpurun_out
for impl in 3xtf32 ffma; do
  timeout 900 python bench.py --steps 30 --warmup 3 --sgemm-impl $impl --no-cpu > $OUT/bench_$impl.log 2>&1; echo "bench $impl rc=$?"
done
BENCH_SMALL="python bench.py --steps 2 --warmup 3 --no-serial --no-e2e --no-cpu --sgemm-impl 3xtf32"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_sgemm_tc -s 1 -c 1 -o $OUT/prof_tc -f $BENCH_SMALL > $OUT/ncu_tc.log 2>&1; echo "ncu tc rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_hist256|k_blackscholes" -s 2 -c 2 -o $OUT/prof_mem2 -f $BENCH_SMALL > $OUT/ncu_mem2.log 2>&1; echo "ncu mem rc=$?"
