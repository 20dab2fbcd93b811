#!/bin/bash
# is the two-logical-GPU gain on one B200 repeatable?  cfg5 as 1, 2 and 4 logical GPUs, alternating
o=gpurun_out/r2c42; mkdir -p $o
for i in 1 2 3; do
  timeout 600 python bench.py --no-serial --no-e2e --no-cpu --no-alt > $o/g1_$i.json 2> $o/g1_$i.err
  SVP_BENCH_DEVICES=0,0 timeout 600 python bench.py --gpus 2 --no-serial --no-e2e --no-cpu --no-alt --no-weak > $o/g2_$i.json 2> $o/g2_$i.err
done
SVP_BENCH_DEVICES=0,0,0,0 timeout 600 python bench.py --gpus 4 --no-serial --no-e2e --no-cpu --no-alt --no-weak > $o/g4_1.json 2> $o/g4_1.err
