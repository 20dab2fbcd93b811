# sized by-value segment tables vs the full 240-segment block, alternating A/B in one session
OUT=gpurun_out
for r in 1 2; do
for full in 0 1; do
  SVP_PARAM_FULL=$full timeout 600 python tools/s1_probe.py > $OUT/s1_probe_full${full}_$r.jsonl 2>&1
  SVP_PARAM_FULL=$full timeout 900 python tools/sweeps.py --only 6 --out $OUT/sweeps_s6_full${full}_$r.json > /dev/null 2>&1
  SVP_PARAM_FULL=$full timeout 900 python bench.py --no-serial --no-alt --no-e2e --no-cpu > $OUT/bench_full${full}_$r.log 2>&1
  echo "full=$full r=$r done"
done
done
