#!/bin/bash
# multi-plan graph cache + bench timed at profile_level 0: graph tests, then cfg1..5 graph 0 vs 1
o=gpurun_out/r2c26; mkdir -p $o
timeout 900 python -m pytest tests/test_gpu_f4.py tests/test_gpu_parity.py -q -p no:cacheprovider -x > $o/pytest_f4_parity.txt 2>&1
for cfg in 1 2 3 4 5; do
  for g in 0 1; do
    timeout 900 python bench.py --config $cfg --no-cpu --no-e2e --graph $g > $o/cfg${cfg}_graph$g.json 2> $o/cfg${cfg}_graph$g.err
  done
done
