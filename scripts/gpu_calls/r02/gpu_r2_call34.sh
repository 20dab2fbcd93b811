#!/bin/bash
# SGEMM epilogue A/B: early accumulator release (all), generic-store epilogue (SVP_TC_EPI=1),
# staggered K-chunk boundaries (SVP_TC_STAGGER=1): parity under each, subnormal fold probe, cfg5 bench
o=gpurun_out/r2c34; mkdir -p $o
for v in "0 0" "1 1"; do
  set -- $v
  SVP_TC_EPI=$1 SVP_TC_STAGGER=$2 timeout 900 python -m pytest tests/test_gpu_sgemm_tc.py tests/test_gpu_sgemm_ieee.py "tests/test_gpu_parity.py::test_config5_sgemm_full_elementwise" -q -p no:cacheprovider -x > $o/pytest_e$1s$2.txt 2>&1
  echo "rc=$?" >> $o/pytest_e$1s$2.txt
done
for e in 0 1; do SVP_TC_EPI=$e timeout 300 python scripts/probe_fold_subnormal.py > $o/probe_e$e.json 2>&1; done
for i in 1 2; do
  for v in "0 0" "1 0" "0 1" "1 1"; do
    set -- $v
    SVP_TC_EPI=$1 SVP_TC_STAGGER=$2 timeout 600 python bench.py --steps 30 --warmup 5 --no-serial --no-e2e --no-cpu --no-alt > $o/bench_e$1s$2_$i.json 2> $o/bench_e$1s$2_$i.err
  done
done
