#!/bin/bash
# device-resident groups split into k launches on k streams (SVP_DEV_SPLIT) vs one launch, vs two
# logical GPUs on the one B200; parity of the cfg5 launch configuration under the split
o=gpurun_out/r2c43; mkdir -p $o
SVP_DEV_SPLIT=2 timeout 900 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -x -k "config5 or config3 or config4" > $o/pytest_split2.txt 2>&1
echo "rc=$?" >> $o/pytest_split2.txt
for i in 1 2; do
  timeout 600 python bench.py --no-serial --no-e2e --no-cpu --no-alt > $o/g1_$i.json 2> $o/g1_$i.err
  SVP_DEV_SPLIT=2 timeout 600 python bench.py --no-serial --no-e2e --no-cpu --no-alt > $o/split2_$i.json 2> $o/split2_$i.err
  SVP_DEV_SPLIT=3 timeout 600 python bench.py --no-serial --no-e2e --no-cpu --no-alt > $o/split3_$i.json 2> $o/split3_$i.err
  SVP_DEV_SPLIT=2 timeout 600 python bench.py --no-serial --no-e2e --no-cpu --no-alt --streams 8 > $o/split2_s8_$i.json 2> $o/split2_s8_$i.err
  SVP_BENCH_DEVICES=0,0 timeout 600 python bench.py --gpus 2 --no-serial --no-e2e --no-cpu --no-alt --no-weak > $o/g2_$i.json 2> $o/g2_$i.err
done
