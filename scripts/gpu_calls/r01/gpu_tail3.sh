# same-box A/B of the tail-when-alone policy: SVP_SGEMM_TAIL=0 vs default, alternating
OUT=gpurun_out
for r in 1 2 3; do for t in 0 1; do
  SVP_SGEMM_TAIL=$t timeout 900 python bench.py --no-serial --no-alt --no-e2e --no-cpu > $OUT/bench_tail3_${t}_$r.log 2>&1
done; done
