#!/bin/bash
# round 2, call 10: K-chunk folds with red.global.add.v4.f32 (no read-back); GPU suite; cfg5 A/B
mkdir -p gpurun_out/r2c10
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/r2c10/pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/r2c10/pytest_gpu.txt
for i in 1 2; do
  for kc in 0 512 1024 256; do
    python bench.py --steps 30 --warmup 5 --no-serial --no-e2e --no-cpu --no-alt --sgemm-kchunk $kc > gpurun_out/r2c10/bench_kc${kc}_$i.json 2> gpurun_out/r2c10/bench_kc${kc}_$i.err
  done
done
python scripts/sgemm_accuracy_seeds.py > gpurun_out/r2c10/accuracy_seeds_default.jsonl 2>/dev/null
