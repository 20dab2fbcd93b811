# sustained-window A/B: default vs hetero (one mixed elementwise launch) vs graph replay
OUT=gpurun_out
for r in 1 2; do
  timeout 900 python bench.py --steps 300 --warmup 10 --no-serial --no-alt --no-e2e --no-cpu > $OUT/bench_susf4_base_$r.log 2>&1
  timeout 900 python bench.py --steps 300 --warmup 10 --no-serial --no-alt --no-e2e --no-cpu --hetero 1 > $OUT/bench_susf4_het_$r.log 2>&1
  timeout 900 python bench.py --steps 300 --warmup 10 --no-serial --no-alt --no-e2e --no-cpu --graph 1 > $OUT/bench_susf4_graph_$r.log 2>&1
done
