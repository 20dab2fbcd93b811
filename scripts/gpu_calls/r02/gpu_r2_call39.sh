#!/bin/bash
# SGEMM stream at the highest priority (SVP_TC_PRIO) with / without cross-flush pipelining
o=gpurun_out/r2c39; mkdir -p $o
for i in 1 2; do
  for v in "0 0" "0 1" "1 0" "1 1"; do
    set -- $v
    SVP_PIPELINE=$1 SVP_TC_PRIO=$2 timeout 600 python bench.py --steps 30 --warmup 5 --no-serial --no-e2e --no-cpu --no-alt > $o/cfg5_pipe$1_prio$2_$i.json 2> $o/cfg5_pipe$1_prio$2_$i.err
  done
done
for v in "0 0" "1 1"; do
  set -- $v
  SVP_PIPELINE=$1 SVP_TC_PRIO=$2 timeout 600 python bench.py --steps 300 --warmup 5 --no-serial --no-e2e --no-cpu --no-alt > $o/cfg5_pipe$1_prio$2_300.json 2> $o/cfg5_pipe$1_prio$2_300.err
done
