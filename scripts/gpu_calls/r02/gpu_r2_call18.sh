#!/bin/bash
# round 2, call 18: 4-deep 8-column epilogue quarter-slabs
mkdir -p gpurun_out/r2c18
timeout 900 python -m pytest tests/test_gpu_sgemm_tc.py tests/test_gpu_sgemm_ieee.py -m gpu -q -p no:cacheprovider > gpurun_out/r2c18/pytest_sgemm.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/r2c18/pytest_sgemm.txt
for i in 1 2; do
  for kc in 0 768 512; do
    python bench.py --steps 30 --warmup 5 --no-serial --no-e2e --no-cpu --no-alt --sgemm-kchunk $kc > gpurun_out/r2c18/bench_kc${kc}_$i.json 2> gpurun_out/r2c18/bench_kc${kc}_$i.err
  done
done
