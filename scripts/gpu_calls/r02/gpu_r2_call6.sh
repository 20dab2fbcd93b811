#!/bin/bash
# round 2, call 6: K-chunked tensor-core accumulation (R23), plain-load SGEMM, GPU suite,
# accuracy vs K / seeds, cfg5 perf A/B over the chunk size
mkdir -p gpurun_out/r2c6
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/r2c6/pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/r2c6/pytest_gpu.txt
python scripts/sgemm_accuracy_k.py > gpurun_out/r2c6/accuracy_k.jsonl 2> gpurun_out/r2c6/accuracy_k.err
python scripts/sgemm_accuracy_seeds.py > gpurun_out/r2c6/accuracy_seeds.jsonl 2> gpurun_out/r2c6/accuracy_seeds.err
for i in 1 2; do
  for kc in 512 0 1024 256; do
    SVP_SGEMM_KCHUNK=$kc python bench.py --steps 30 --warmup 5 --no-serial --no-e2e --no-cpu --no-alt > gpurun_out/r2c6/bench_kc${kc}_$i.json 2> gpurun_out/r2c6/bench_kc${kc}_$i.err
  done
done
