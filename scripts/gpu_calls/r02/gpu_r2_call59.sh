#!/bin/bash
# DMMA 32x32 tiles for every DGEMM launch (big ones too); SIMT kernels kept under SVP_DGEMM_DMMA=0
o=gpurun_out/r2c59; mkdir -p $o
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "dgemm or table1" > $o/pytest_dgemm.txt 2>&1
echo "rc=$?" >> $o/pytest_dgemm.txt
timeout 900 python tools/sweeps.py --only 5 --out $o/s5_dmma_all.json > $o/s5.log 2>&1
SVP_DGEMM_DMMA=0 timeout 900 python tools/sweeps.py --only 5 --out $o/s5_simt.json > $o/s5_simt.log 2>&1
