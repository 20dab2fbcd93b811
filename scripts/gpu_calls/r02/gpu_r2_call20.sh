#!/bin/bash
# S6 launch-bound mix: HEAD vs the round-1 tree (abtree/r1, built lib), alternating, 3x each.
mkdir -p gpurun_out/r2c20
for i in 1 2 3; do
  timeout 600 python tools/sweeps.py --only 6 --out gpurun_out/r2c20/head_$i.json > gpurun_out/r2c20/head_$i.log 2>&1
  (cd abtree/r1 && timeout 600 python tools/sweeps.py --only 6 --out ../../gpurun_out/r2c20/r1_$i.json > ../../gpurun_out/r2c20/r1_$i.log 2>&1)
done
