#!/bin/bash
# round 2, call 3: exact recompute of NaN accumulators -- GPU suite + A/B vs the round-1 SGEMM
mkdir -p gpurun_out/r2c3
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/r2c3/pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/r2c3/pytest_gpu.txt
python scripts/ieee_probe.py > gpurun_out/r2c3/ieee_probe.jsonl 2>/dev/null
for i in 1 2; do
  python bench.py --steps 30 --warmup 5 --no-serial --no-e2e --no-cpu --no-alt > gpurun_out/r2c3/bench_new_$i.json 2> gpurun_out/r2c3/bench_new_$i.err
  SVP_LIB=ab_libs/libsvp_oldconv.so python bench.py --steps 30 --warmup 5 --no-serial --no-e2e --no-cpu --no-alt > gpurun_out/r2c3/bench_old_$i.json 2> gpurun_out/r2c3/bench_old_$i.err
done
