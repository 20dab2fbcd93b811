#!/bin/bash
# dynamic SGEMM tile order (SVP_TC_DYN) + pipelined TMEM reads in the epilogue (SVP_TC_EPI_PF):
# full GPU suite at the new defaults, then same-box A/B of cfg5 (timed step and one-stream SGEMM)
o=gpurun_out/r2c36; mkdir -p $o
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider -x > $o/pytest_gpu.txt 2>&1
echo "rc=$?" >> $o/pytest_gpu.txt
for i in 1 2; do
  for v in "1 1" "0 1" "1 0" "0 0"; do
    set -- $v
    SVP_TC_DYN=$1 SVP_TC_EPI_PF=$2 timeout 600 python bench.py --steps 30 --warmup 5 --no-serial --no-e2e --no-cpu --no-alt > $o/bench_dyn$1_pf$2_$i.json 2> $o/bench_dyn$1_pf$2_$i.err
  done
done
