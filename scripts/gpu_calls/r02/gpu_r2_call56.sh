#!/bin/bash
# small DGEMM: A fragments as LDS.128 (rows padded to TM+2) vs HEAD (libsvp_head.so), Table 1 sweep
o=gpurun_out/r2c56; mkdir -p $o
timeout 900 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "dgemm or table1" > $o/pytest_dgemm.txt 2>&1
echo "rc=$?" >> $o/pytest_dgemm.txt
for i in 1 2; do
  timeout 900 python tools/sweeps.py --only 5 --out $o/s5_new_$i.json > $o/s5_new_$i.log 2>&1
  SVP_LIB=$PWD/paper_conf_dac_jungc15_b200/libsvp_head.so timeout 900 python tools/sweeps.py --only 5 --out $o/s5_head_$i.json > $o/s5_head_$i.log 2>&1
done
