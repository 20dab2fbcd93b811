#!/bin/bash
# split-K small DGEMM on clusters (DSMEM reduction in rank order): DGEMM parity, then the Table 1
# program sweep (S5) with the split on / off
o=gpurun_out/r2c52; mkdir -p $o
timeout 900 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "dgemm or table1 or Table1" > $o/pytest_dgemm.txt 2>&1
echo "rc=$?" >> $o/pytest_dgemm.txt
for v in 1 0; do
  SVP_DGEMM_SPLIT=$v timeout 900 python tools/sweeps.py --only 5 --out $o/s5_split$v.json > $o/s5_split$v.log 2>&1
done
