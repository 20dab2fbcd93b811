# sustained-window A/B: resident CTAs/SM of the memory-bound launches (energy at the power cap)
OUT=gpurun_out
for r in 1 2; do
  timeout 900 python bench.py --steps 300 --warmup 10 --no-serial --no-alt --no-e2e --no-cpu > $OUT/bench_susg_base_$r.log 2>&1
  SVP_EW_PER_SM=3 SVP_BS_PER_SM=2 timeout 900 python bench.py --steps 300 --warmup 10 --no-serial --no-alt --no-e2e --no-cpu > $OUT/bench_susg_low_$r.log 2>&1
done
