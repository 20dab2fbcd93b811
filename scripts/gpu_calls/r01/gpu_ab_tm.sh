OUT=gpurun_out
for r in 1 2 3; do for tm in 0 1; do
  timeout 300 python bench.py --steps 30 --warmup 3 --no-e2e --no-cpu --no-serial --no-alt --table-mode $tm > $OUT/bench_ab_tm${tm}_$r.log 2>&1; echo "r=$r tm=$tm rc=$?"
done; done
