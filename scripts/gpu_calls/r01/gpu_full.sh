# full round-end style pass: GPU tests, smoke, full bench (default flags), ncu launch list + captures
OUT=gpurun_out
timeout 1500 python -m pytest tests -m gpu -q --timeout 300 -p no:cacheprovider > $OUT/pytest_gpu_full.log 2>&1; echo "pytest rc=$?"; tail -2 $OUT/pytest_gpu_full.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?"
timeout 1200 python bench.py > $OUT/bench_full.log 2>&1; echo "bench rc=$?"
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > $OUT/bench_ref.log 2>&1; echo "ref rc=$?"
BENCH_SMALL="python bench.py --steps 2 --warmup 3 --no-serial --no-e2e --no-cpu --no-alt"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:k_ --csv --log-file $OUT/launches.csv $BENCH_SMALL > $OUT/ncu_launches.log 2>&1; echo "ncu list rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_sgemm_tc|k_vecadd|k_saxpy|k_hist256|k_blackscholes" -s 5 -c 5 -o $OUT/prof_full -f $BENCH_SMALL > $OUT/ncu_full.log 2>&1; echo "ncu full rc=$?"
