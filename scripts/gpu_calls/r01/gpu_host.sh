# planner/submit host-path speedups: GPU tests, S6 launch-bound mixes, S1 probe, default bench
OUT=gpurun_out
timeout 1500 python -m pytest tests -m gpu -q --timeout 300 -p no:cacheprovider > $OUT/pytest_gpu_host.log 2>&1; echo "pytest rc=$?"; tail -2 $OUT/pytest_gpu_host.log
for r in 1 2; do timeout 900 python tools/sweeps.py --only 6 --out $OUT/sweeps_s6_host_$r.json > /dev/null 2>&1; done
timeout 600 python tools/s1_probe.py > $OUT/s1_probe_host.jsonl 2>&1; echo "s1 rc=$?"
timeout 1200 python bench.py > $OUT/bench_host.log 2>&1; echo "bench rc=$?"
