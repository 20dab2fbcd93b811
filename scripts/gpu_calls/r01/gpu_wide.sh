# wide (256x512) TF32+2xBF16 pair tiles: parity, then A/B timing vs 256x256 and energy
OUT=gpurun_out
timeout 900 python -m pytest tests/test_gpu_sgemm_tc.py tests/test_gpu_parity.py -m gpu -q --timeout 600 -p no:cacheprovider -k "sgemm or config5 or tc" > $OUT/t_wide.log 2>&1; echo "pytest rc=$?"; tail -3 $OUT/t_wide.log
: > $OUT/energy_wide.jsonl
for i in 1 2; do
timeout 120 env SVP_TC_WIDE=1 python scripts/energy_probe.py sgemm 2 wide >> $OUT/energy_wide.jsonl 2>>$OUT/energy_wide.err
timeout 120 env SVP_TC_WIDE=0 python scripts/energy_probe.py sgemm 2 pair256 >> $OUT/energy_wide.jsonl 2>>$OUT/energy_wide.err
done
cat $OUT/energy_wide.jsonl
for i in 1 2; do
SVP_TC_WIDE=1 timeout 600 python bench.py --no-serial --no-e2e --no-cpu --no-alt > $OUT/bench_wide_$i.log 2>&1
SVP_TC_WIDE=0 timeout 600 python bench.py --no-serial --no-e2e --no-cpu --no-alt > $OUT/bench_pair256_$i.log 2>&1
done
for f in $OUT/bench_wide_*.log $OUT/bench_pair256_*.log; do tail -1 $f | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$f', round(d['value']), round(d['ms_per_step'],3), round(d['roofline']['achieved'],1), d['clocks']['sm_mhz'])"; done
