#!/bin/bash
# vecadd dynamic order, take 2: only for launches with >= 4 tiles per resident CTA; is the
# profile_level-2 split test sensitive to the DYN-compiled vecadd kernel?
o=gpurun_out/r2c50; mkdir -p $o
for i in 1 2 3; do
  for v in 0 1; do
    SVP_VECADD_DYN=$v timeout 300 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "measured_split_level2" > $o/pytest_l2_dyn${v}_$i.txt 2>&1
    echo "rc=$?" >> $o/pytest_l2_dyn${v}_$i.txt
  done
done
for v in 0 1; do
  SVP_VECADD_DYN=$v timeout 600 python bench.py --config 1 --steps 300 --warmup 20 --no-serial --no-e2e --no-cpu --no-alt > $o/cfg1_dyn${v}.json 2> $o/cfg1_dyn${v}.err
  SVP_VECADD_DYN=$v timeout 600 python bench.py --config 4 --steps 100 --warmup 10 --no-serial --no-e2e --no-cpu --no-alt > $o/cfg4_dyn${v}.json 2> $o/cfg4_dyn${v}.err
done
