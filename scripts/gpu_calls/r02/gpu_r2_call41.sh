#!/bin/bash
# launch-bound BASELINE configs over longer windows (a 30-step window of ~10 us steps is 0.3 ms):
# full bench lines for cfg1 / cfg2 at 300 steps (serial baselines 60 steps), cfg3 / cfg4 at 100
o=gpurun_out/r2c41; mkdir -p $o
for c in 1 2; do
  timeout 900 python bench.py --config $c --steps 300 --warmup 20 > $o/bench_cfg${c}_300.json 2> $o/bench_cfg${c}_300.err
done
for c in 3 4; do
  timeout 900 python bench.py --config $c --steps 100 --warmup 10 > $o/bench_cfg${c}_100.json 2> $o/bench_cfg${c}_100.err
done
