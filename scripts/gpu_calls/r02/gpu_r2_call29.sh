#!/bin/bash
# bench passes after a 1 s rest: cfg5 default x2 and --timed-profile-level 1 x1 (iso SGEMM should be ~2.64 ms again)
o=gpurun_out/r2c29; mkdir -p $o
for i in 1 2; do
  timeout 600 python bench.py --no-cpu --no-e2e > $o/head_rest_$i.json 2> $o/head_rest_$i.err
done
timeout 600 python bench.py --no-cpu --no-e2e --timed-profile-level 1 > $o/head_rest_p1.json 2> $o/head_rest_p1.err
