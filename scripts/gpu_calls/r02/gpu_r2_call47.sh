#!/bin/bash
# TMA multicast vs unicast L2 traffic at cluster sizes 1/2/4 (tools/tma_mc_probe.cu)
o=gpurun_out/r2c47; mkdir -p $o
nvcc -gencode arch=compute_100a,code=sm_100a -O2 -lineinfo -o /tmp/tma_mc_probe tools/tma_mc_probe.cu > $o/build.txt 2>&1
for v in "1 uc" "2 uc" "2 mc" "4 uc" "4 mc"; do
  set -- $v
  timeout 60 /tmp/tma_mc_probe $1 $2 2000 >> $o/probe.jsonl 2>> $o/probe.err
done
for v in "1 uc" "2 uc" "2 mc" "4 uc" "4 mc"; do
  set -- $v
  timeout 300 ncu --metrics gpu__time_duration.sum,lts__t_bytes.sum,lts__t_sectors_op_read.sum,lts__t_requests_op_read.sum,lts__t_sectors_srcunit_tex_op_read.sum,dram__bytes_read.sum \
     --clock-control none -s 1 -c 1 --csv --log-file $o/ncu_cs$1_$2.csv /tmp/tma_mc_probe $1 $2 2000 > $o/ncu_cs$1_$2.log 2>&1
done
timeout 300 ncu --set full --clock-control none -s 1 -c 1 -o $o/full_cs4_mc /tmp/tma_mc_probe 4 mc 2000 > $o/full_cs4_mc.log 2>&1
timeout 300 ncu --set full --clock-control none -s 1 -c 1 -o $o/full_cs4_uc /tmp/tma_mc_probe 4 uc 2000 > $o/full_cs4_uc.log 2>&1
