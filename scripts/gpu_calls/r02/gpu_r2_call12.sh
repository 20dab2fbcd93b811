#!/bin/bash
# round 2, call 12: TMA epilogue for every beta == 0 tensor-core SGEMM tile; hist claim-ahead
mkdir -p gpurun_out/r2c12
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/r2c12/pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/r2c12/pytest_gpu.txt
for i in 1 2; do
  for kc in 0 512 768 1024; do
    python bench.py --steps 30 --warmup 5 --no-serial --no-e2e --no-cpu --no-alt --sgemm-kchunk $kc > gpurun_out/r2c12/bench_kc${kc}_$i.json 2> gpurun_out/r2c12/bench_kc${kc}_$i.err
  done
  SVP_HIST_DYN=0 python bench.py --steps 30 --warmup 5 --no-serial --no-e2e --no-cpu --no-alt > gpurun_out/r2c12/bench_histstatic_$i.json 2> gpurun_out/r2c12/bench_histstatic_$i.err
done
for kc in 512 768 1024; do ACC_KCHUNK=$kc python scripts/sgemm_accuracy_seeds.py > gpurun_out/r2c12/accuracy_seeds_kc$kc.jsonl 2>/dev/null; done
