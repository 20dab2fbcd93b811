# least-loaded compute streams vs round-robin: alternating bench A/B + plan check
OUT=gpurun_out
for r in 1 2 3; do for rr in 1 0; do
  SVP_STREAM_RR=$rr timeout 900 python bench.py --no-serial --no-alt --no-e2e --no-cpu > $OUT/bench_rr${rr}_$r.log 2>&1
done; done
