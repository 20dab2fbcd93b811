OUT=gpurun_out
for a in 8 16 24; do
  timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu --no-serial --no-alt --arena-gb $a > $OUT/bench_e2e_a$a.log 2>&1; echo "arena=$a rc=$?"
done
SVP_BENCH_MAXCH=16 timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu --no-serial --no-alt --arena-gb 16 > $OUT/bench_e2e_a16_c16.log 2>&1; echo "arena=16 ch16 rc=$?"
