# Black-Scholes: parity after the SFU change, then tile-shape variants (kBsVec) rebuilt on the box
OUT=gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_f4.py -m gpu -q --timeout 600 -p no:cacheprovider -k "mixed_small or config4 or config3 or hetero" > $OUT/t_bs.log 2>&1; echo "pytest rc=$?"; tail -1 $OUT/t_bs.log
: > $OUT/bs_vec.jsonl
cp paper_conf_dac_jungc15_b200/csrc/tables.h /tmp/tables.h.orig
for V in 2 1 4; do
  sed -i "s/constexpr int kBsVec = [0-9];/constexpr int kBsVec = $V;/" paper_conf_dac_jungc15_b200/csrc/tables.h
  python -c "from paper_conf_dac_jungc15_b200 import _build; _build.build()" > /dev/null 2>&1 || echo "build V=$V failed"
  timeout 300 python tools/grid_probe.py blackscholes,all 2>&1 | grep RESULT | sed "s/^RESULT /V$V /" >> $OUT/bs_vec.jsonl
done
cp /tmp/tables.h.orig paper_conf_dac_jungc15_b200/csrc/tables.h
cat $OUT/bs_vec.jsonl | cut -c1-220
