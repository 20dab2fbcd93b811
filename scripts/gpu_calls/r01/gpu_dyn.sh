# dynamic tile order for Black-Scholes: GPU tests, alternating bench A/B, ncu balance
OUT=gpurun_out
timeout 1500 python -m pytest tests -m gpu -q --timeout 300 -p no:cacheprovider > $OUT/pytest_gpu_dyn.log 2>&1; echo "pytest rc=$?"; tail -2 $OUT/pytest_gpu_dyn.log
for r in 1 2 3; do for dyn in 0 1; do
  SVP_EW_DYN=$dyn timeout 900 python bench.py --no-serial --no-alt --no-e2e --no-cpu > $OUT/bench_dyn${dyn}_$r.log 2>&1
done; done
BENCH_SMALL="python bench.py --steps 2 --warmup 3 --no-serial --no-e2e --no-cpu --no-alt"
for dyn in 0 1; do
SVP_EW_DYN=$dyn timeout 600 ncu --metrics gpu__time_duration.sum,sm__cycles_active.min,sm__cycles_active.avg,sm__cycles_active.max,gpc__cycles_elapsed.max,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:k_blackscholes -c 3 --csv --log-file $OUT/ncu_bs_dyn$dyn.csv $BENCH_SMALL > /dev/null 2>&1; echo "ncu $dyn rc=$?"
done
