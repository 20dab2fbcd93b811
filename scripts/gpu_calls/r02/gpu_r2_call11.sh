#!/bin/bash
# round 2, call 11: K-chunk folds through TMA store / reduce-add; hist256 dynamic order; GPU suite + A/B
mkdir -p gpurun_out/r2c11
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/r2c11/pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/r2c11/pytest_gpu.txt
for i in 1 2; do
  for kc in 0 512 1024; do
    python bench.py --steps 30 --warmup 5 --no-serial --no-e2e --no-cpu --no-alt --sgemm-kchunk $kc > gpurun_out/r2c11/bench_kc${kc}_$i.json 2> gpurun_out/r2c11/bench_kc${kc}_$i.err
  done
  SVP_HIST_DYN=0 python bench.py --steps 30 --warmup 5 --no-serial --no-e2e --no-cpu --no-alt > gpurun_out/r2c11/bench_histstatic_$i.json 2> gpurun_out/r2c11/bench_histstatic_$i.err
done
SVP_SGEMM_KCHUNK=512 python scripts/sgemm_accuracy_seeds.py > gpurun_out/r2c11/accuracy_seeds_kc512.jsonl 2>/dev/null
