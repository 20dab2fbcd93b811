#!/bin/bash
# SGEMM tile shape under K chunks: wide 256x512 pair tiles (one TMEM accumulator, SVP_TC_WIDE=1)
# vs 256x256 pair tiles (two accumulators, drains overlap the next unit's MMAs; SVP_TC_WIDE=0),
# at the default 768-k chunks and unchunked; cfg5 bench, alternating
o=gpurun_out/r2c24; mkdir -p $o
for i in 1 2; do
  for w in 1 0; do
    for kc in 768 0; do
      SVP_TC_WIDE=$w timeout 600 python bench.py --steps 20 --warmup 3 --no-serial --no-alt --no-cpu --no-e2e \
        --sgemm-kchunk $kc > $o/wide${w}_kc${kc}_$i.json 2> $o/wide${w}_kc${kc}_$i.err
    done
  done
done
