#!/bin/bash
# launch-bound configs (cfg1 2 VPs, cfg2 16 x SGEMM 512^3): timed-arm profile_level 1 vs 0,
# graph 0 vs 1; plus the long-K chunk-16 parity case
o=gpurun_out/r2c25; mkdir -p $o
for cfg in 1 2; do
  for prof in 1 0; do
    for g in 0 1; do
      SVP_BENCH_TIMED_PROF=$prof timeout 600 python bench.py --config $cfg --steps 200 --warmup 20 --no-alt --no-cpu --no-e2e \
        --graph $g > $o/cfg${cfg}_prof${prof}_graph$g.json 2> $o/cfg${cfg}_prof${prof}_graph$g.err
    done
  done
done
timeout 600 python -m pytest tests/test_gpu_sgemm_tc.py -k "long_k" -q -p no:cacheprovider > $o/pytest_longk.txt 2>&1
