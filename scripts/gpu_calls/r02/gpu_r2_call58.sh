#!/bin/bash
# small DGEMM tiles on the FP64 tensor cores (mma.sync m8n8k4 DMMA, SVP_DGEMM_DMMA): parity, S5 A/B
o=gpurun_out/r2c58; mkdir -p $o
timeout 900 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "dgemm or table1" > $o/pytest_dgemm.txt 2>&1
echo "rc=$?" >> $o/pytest_dgemm.txt
SVP_DGEMM_SPLIT=0 timeout 900 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "dgemm or table1" > $o/pytest_dgemm_nosplit.txt 2>&1
echo "rc=$?" >> $o/pytest_dgemm_nosplit.txt
for i in 1 2; do
  for v in 1 0; do
    SVP_DGEMM_DMMA=$v timeout 900 python tools/sweeps.py --only 5 --out $o/s5_dmma${v}_$i.json > $o/s5_dmma${v}_$i.log 2>&1
  done
done
