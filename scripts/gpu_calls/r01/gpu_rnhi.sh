# 4xBF16 split (SVP_TC_RNHI=1) vs TF32+2xBF16: parity (forced wide and 256x256), accuracy, energy, bench
OUT=gpurun_out
for w in 2 0; do
SVP_TC_RNHI=1 SVP_TC_WIDE=$w timeout 900 python -m pytest tests/test_gpu_sgemm_tc.py tests/test_gpu_parity.py -m gpu -q --timeout 600 -p no:cacheprovider -k "(fp32_tolerance or ragged_alpha_beta or wide_dynamic or 2048_sampled or config5) and not variants" > $OUT/t_rnhi_w$w.log 2>&1; echo "pytest wide=$w rc=$?"; tail -1 $OUT/t_rnhi_w$w.log
done
SVP_TC_RNHI=1 timeout 300 python scripts/sgemm_accuracy.py > $OUT/acc_rnhi.json 2>&1; python -c "import json; d=json.load(open('$OUT/acc_rnhi.json')); print('rnhi acc', d['tf32bf16'])"
: > $OUT/energy_rnhi.jsonl
for i in 1 2; do
timeout 120 env SVP_TC_RNHI=1 python scripts/energy_probe.py sgemm 2 rnhi >> $OUT/energy_rnhi.jsonl 2>>$OUT/energy_rnhi.err
timeout 120 env SVP_TC_RNHI=0 python scripts/energy_probe.py sgemm 2 tf32bf16 >> $OUT/energy_rnhi.jsonl 2>>$OUT/energy_rnhi.err
done
cat $OUT/energy_rnhi.jsonl
for i in 1 2; do
SVP_TC_RNHI=1 timeout 600 python bench.py --no-serial --no-e2e --no-cpu --no-alt > $OUT/bench_rnhi_$i.log 2>&1
SVP_TC_RNHI=0 timeout 600 python bench.py --no-serial --no-e2e --no-cpu --no-alt > $OUT/bench_tf32bf16_$i.log 2>&1
done
for f in $OUT/bench_rnhi_*.log $OUT/bench_tf32bf16_*.log; do tail -1 $f | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$f', round(d['value']), round(d['ms_per_step'],3), round(d['roofline']['achieved'],1), d['clocks']['sm_mhz'])"; done
