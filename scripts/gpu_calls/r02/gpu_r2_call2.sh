#!/bin/bash
# round 2, call 2: IEEE converter changes -- GPU suite + converter A/B on the cfg5 bench
mkdir -p gpurun_out/r2c2
timeout 1700 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/r2c2/pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/r2c2/pytest_gpu.txt
for i in 1 2; do
  python bench.py --steps 30 --warmup 5 --no-serial --no-e2e --no-cpu --no-alt > gpurun_out/r2c2/bench_new_$i.json 2> gpurun_out/r2c2/bench_new_$i.err
  SVP_LIB=ab_libs/libsvp_oldconv.so python bench.py --steps 30 --warmup 5 --no-serial --no-e2e --no-cpu --no-alt > gpurun_out/r2c2/bench_old_$i.json 2> gpurun_out/r2c2/bench_old_$i.err
done
python bench.py --steps 30 --warmup 5 --no-serial --no-e2e --no-cpu > gpurun_out/r2c2/bench_new_alt.json 2> gpurun_out/r2c2/bench_new_alt.err
