#!/bin/bash
# split-K DGEMM take 2: split variants capped at 168 registers (6 CTAs/SM), the unsplit variants
# back to their own register budgets; DGEMM parity, S5 split on / off
o=gpurun_out/r2c54; mkdir -p $o
timeout 900 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "dgemm or table1" > $o/pytest_dgemm.txt 2>&1
echo "rc=$?" >> $o/pytest_dgemm.txt
for v in 1 0; do
  SVP_DGEMM_SPLIT=$v timeout 900 python tools/sweeps.py --only 5 --out $o/s5_split$v.json > $o/s5_split$v.log 2>&1
done
