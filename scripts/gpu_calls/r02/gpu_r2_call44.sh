#!/bin/bash
# randomized async flush sequences with mixed residency and a wrapping arena, against the oracle
o=gpurun_out/r2c44; mkdir -p $o
timeout 900 python -m pytest tests/test_gpu_fuzz.py -q -p no:cacheprovider > $o/pytest_fuzz.txt 2>&1
echo "rc=$?" >> $o/pytest_fuzz.txt
