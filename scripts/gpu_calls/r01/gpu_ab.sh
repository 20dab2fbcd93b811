OUT=gpurun_out
for cs in 1 0; do
  SVP_COSCHEDULE=$cs timeout 600 python bench.py --steps 30 --warmup 3 --no-e2e --no-cpu --no-serial --no-alt > $OUT/bench_cs$cs.log 2>&1; echo "cs=$cs rc=$?"
done
