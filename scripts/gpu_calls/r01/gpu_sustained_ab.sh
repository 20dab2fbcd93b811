# sustained-window (300 steps, board at the power cap) A/B of this session's neutral switches
OUT=gpurun_out
for r in 1 2; do
  for cfg in "base" "SVP_HIST_FUSED=1" "SVP_STREAM_RR=1"; do
    if [ "$cfg" = base ]; then e=""; else e="$cfg"; fi
    env $e timeout 900 python bench.py --steps 300 --warmup 10 --no-serial --no-alt --no-e2e --no-cpu > $OUT/bench_sus_${cfg//=/_}_$r.log 2>&1
  done
done
