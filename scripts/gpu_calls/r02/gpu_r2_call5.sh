#!/bin/bash
# round 2, call 5: hist256 warp-adaptive tables, sgemm K routing (R23); GPU suite; hist A/B;
# K=2048 accuracy margin; bench --gpus 2 (logical) path; e2e timeline
mkdir -p gpurun_out/r2c5
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/r2c5/pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/r2c5/pytest_gpu.txt
for i in 1 2; do
  python bench.py --steps 30 --warmup 5 --no-serial --no-e2e --no-cpu --no-alt > gpurun_out/r2c5/bench_new_$i.json 2> gpurun_out/r2c5/bench_new_$i.err
  SVP_LIB=ab_libs/libsvp_hist_r1.so python bench.py --steps 30 --warmup 5 --no-serial --no-e2e --no-cpu --no-alt > gpurun_out/r2c5/bench_histr1_$i.json 2> gpurun_out/r2c5/bench_histr1_$i.err
done
python scripts/sgemm_accuracy_seeds.py > gpurun_out/r2c5/accuracy_seeds.jsonl 2> gpurun_out/r2c5/accuracy_seeds.err
SVP_BENCH_DEVICES=0,0 timeout 600 python bench.py --gpus 2 --steps 10 --warmup 3 --no-serial --no-alt --no-cpu --no-e2e > gpurun_out/r2c5/bench_gpus2_logical.json 2> gpurun_out/r2c5/bench_gpus2_logical.err
timeout 600 python tools/e2e_timeline.py --out gpurun_out/r2c5/e2e_timeline.json > gpurun_out/r2c5/e2e_timeline.log 2>&1
