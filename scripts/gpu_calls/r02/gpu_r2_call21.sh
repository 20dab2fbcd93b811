#!/bin/bash
# host-path phases of S6's launch-bound mix: HEAD (bucket from exponent bits, one elapsed query
# per op) vs the round-1 tree, alternating
mkdir -p gpurun_out/r2c21
for i in 1 2; do
  timeout 300 python tools/host_phases.py --out gpurun_out/r2c21/head_$i.json > gpurun_out/r2c21/head_$i.log 2>&1
  (cd abtree/r1 && timeout 300 python tools/host_phases.py --out ../../gpurun_out/r2c21/r1_$i.json > ../../gpurun_out/r2c21/r1_$i.log 2>&1)
done
