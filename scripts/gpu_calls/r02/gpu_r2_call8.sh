#!/bin/bash
# round 2, call 8: GPU suite (K-chunk + plain sgemm), cfg5 A/B over chunking x wide, mode-H stream study
mkdir -p gpurun_out/r2c8
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/r2c8/pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/r2c8/pytest_gpu.txt
for i in 1 2; do
  for cfg in "512 1" "0 1" "512 0" "0 0" "1024 1"; do
    set -- $cfg
    SVP_SGEMM_KCHUNK=$1 SVP_TC_WIDE=$2 python bench.py --steps 30 --warmup 5 --no-serial --no-e2e --no-cpu --no-alt > gpurun_out/r2c8/bench_kc$1_w$2_$i.json 2> gpurun_out/r2c8/bench_kc$1_w$2_$i.err
  done
done
python tools/e2e_timeline.py --out gpurun_out/r2c8/tl_default.json > gpurun_out/r2c8/tl.log 2>&1
SVP_FIRST_COMPUTE_STREAM=1 python tools/e2e_timeline.py --streams 5 --out gpurun_out/r2c8/tl_skip0.json >> gpurun_out/r2c8/tl.log 2>&1
