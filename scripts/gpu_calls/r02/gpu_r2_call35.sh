#!/bin/bash
# same-box A/B: SGEMM epilogue early accumulator release (SVP_TC_EARLY=1, default) vs release after the last write
o=gpurun_out/r2c35; mkdir -p $o
timeout 600 python -m pytest tests/test_gpu_sgemm_tc.py "tests/test_gpu_parity.py::test_config5_sgemm_full_elementwise" -q -p no:cacheprovider -x > $o/pytest.txt 2>&1
echo "rc=$?" >> $o/pytest.txt
for i in 1 2 3; do
  for e in 0 1; do
    SVP_TC_EARLY=$e timeout 600 python bench.py --steps 30 --warmup 5 --no-serial --no-e2e --no-cpu --no-alt > $o/bench_early${e}_$i.json 2> $o/bench_early${e}_$i.err
  done
done
