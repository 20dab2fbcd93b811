# hist256 ragged tiles through the ring: GPU tests, hist probe, ncu balance of the cfg5 hist launch
OUT=gpurun_out
timeout 1500 python -m pytest tests -m gpu -q --timeout 300 -p no:cacheprovider > $OUT/pytest_gpu_hist.log 2>&1; echo "pytest rc=$?"; tail -3 $OUT/pytest_gpu_hist.log
timeout 300 python tools/hist_probe.py $OUT/hist_probe2.json > $OUT/hist_probe2.log 2>&1; cat $OUT/hist_probe2.log
BENCH_SMALL="python bench.py --steps 2 --warmup 3 --no-serial --no-e2e --no-cpu --no-alt"
timeout 600 ncu --metrics gpu__time_duration.sum,sm__cycles_active.min,sm__cycles_active.avg,sm__cycles_active.max,gpc__cycles_elapsed.max,dram__bytes_read.sum --clock-control none -k regex:k_hist256 -c 3 --csv --log-file $OUT/ncu_hist.csv $BENCH_SMALL > /dev/null 2>&1; echo "ncu rc=$?"
python - <<'PY'
import csv
rows=list(csv.reader(open('gpurun_out/ncu_hist.csv')))
hi=[i for i,r in enumerate(rows) if 'Metric Name' in r][0]; h=rows[hi]
for r in rows[hi+1:]:
    d=dict(zip(h,r)); print(d['Kernel Name'][:20], d['Metric Name'], d['Metric Value'])
PY
