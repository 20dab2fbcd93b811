# single-launch hist256: GPU tests, hist probe A/B, bench A/B
OUT=gpurun_out
timeout 1500 python -m pytest tests -m gpu -q --timeout 300 -p no:cacheprovider > $OUT/pytest_gpu_hf.log 2>&1; echo "pytest rc=$?"; tail -2 $OUT/pytest_gpu_hf.log
for f in 0 1; do SVP_HIST_FUSED=$f timeout 300 python tools/hist_probe.py $OUT/hist_probe_fused$f.json > /dev/null 2>&1; echo "probe $f"; cat $OUT/hist_probe_fused$f.json | tr -d '\n' | cut -c1-400; echo; done
for r in 1 2; do for f in 0 1; do
  SVP_HIST_FUSED=$f timeout 900 python bench.py --no-serial --no-alt --no-e2e --no-cpu > $OUT/bench_hf${f}_$r.log 2>&1
done; done
