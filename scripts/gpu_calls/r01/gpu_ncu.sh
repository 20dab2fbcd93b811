# ncu evidence for the current default path: launch list of the bench command + one full capture per kernel
OUT=gpurun_out
BENCH_SMALL="python bench.py --steps 2 --warmup 3 --no-serial --no-e2e --no-cpu --no-alt"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:k_ --csv --log-file $OUT/launches.csv $BENCH_SMALL > $OUT/ncu_launches.log 2>&1; echo "ncu list rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_sgemm_tc|k_vecadd|k_saxpy|k_hist256|k_blackscholes" -s 5 -c 5 -o $OUT/prof_full -f $BENCH_SMALL > $OUT/ncu_full.log 2>&1; echo "ncu full rc=$?"
ls -la $OUT/prof_full.ncu-rep
