#!/bin/bash
# cfg5 one-stream SGEMM time (the roofline figure) across bench variants on ONE box, alternating:
# HEAD default / HEAD --graph 0 / HEAD --timed-profile-level 1 --graph 0 / tree at 7c62cb0 (before the graph default)
o=gpurun_out/r2c28; mkdir -p $o
for i in 1 2; do
  timeout 600 python bench.py --no-serial --no-alt --no-cpu --no-e2e > $o/head_default_$i.json 2> $o/head_default_$i.err
  timeout 600 python bench.py --no-serial --no-alt --no-cpu --no-e2e --graph 0 > $o/head_g0_$i.json 2> $o/head_g0_$i.err
  timeout 600 python bench.py --no-serial --no-alt --no-cpu --no-e2e --graph 0 --timed-profile-level 1 > $o/head_g0p1_$i.json 2> $o/head_g0p1_$i.err
  (cd abtree/r2a && timeout 600 python bench.py --no-serial --no-alt --no-cpu --no-e2e > ../../$o/old_$i.json 2> ../../$o/old_$i.err)
done
