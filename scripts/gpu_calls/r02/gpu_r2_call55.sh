#!/bin/bash
# where the small DGEMM's time goes: ncu --set full of one Table 1 level launch (8 VPs, 800 32x32 tiles)
o=gpurun_out/r2c55; mkdir -p $o
timeout 300 python scripts/dgemm_table1_probe.py 8 4 > $o/probe.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_dgemm -s 8 -c 1 -o $o/dgemm8 python scripts/dgemm_table1_probe.py 8 4 > $o/ncu8.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_dgemm -s 8 -c 1 -o $o/dgemm1 python scripts/dgemm_table1_probe.py 1 4 > $o/ncu1.log 2>&1
