#!/bin/bash
# with the default 768-k chunks: wide 256x512 pair tiles (one accumulator set, exposed drains at
# chunk boundaries) vs narrow 256x256 pair tiles (two TMEM accumulators ping-pong across chunks)
o=gpurun_out/r2c45; mkdir -p $o
for i in 1 2 3; do
  for w in 1 0; do
    SVP_TC_WIDE=$w timeout 600 python bench.py --no-serial --no-e2e --no-cpu --no-alt > $o/wide${w}_$i.json 2> $o/wide${w}_$i.err
  done
done
