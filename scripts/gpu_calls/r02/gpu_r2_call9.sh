#!/bin/bash
# round 2, call 9: control stream split, sgemm_kchunk config; GPU suite; full bench lines for
# BASELINE configs 1-5; mode-H timeline; Black-Scholes error report
mkdir -p gpurun_out/r2c9
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/r2c9/pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/r2c9/pytest_gpu.txt
python bench.py > gpurun_out/r2c9/bench_cfg5.json 2> gpurun_out/r2c9/bench_cfg5.err
for c in 1 2 3 4; do
  python bench.py --config $c > gpurun_out/r2c9/bench_cfg$c.json 2> gpurun_out/r2c9/bench_cfg$c.err
done
python tools/e2e_timeline.py --out gpurun_out/r2c9/tl_default.json > gpurun_out/r2c9/tl.log 2>&1
python tools/e2e_timeline.py --profile 0 >> gpurun_out/r2c9/tl.log 2>&1
python scripts/bs_error.py --out gpurun_out/r2c9/bs_error.json > gpurun_out/r2c9/bs_error.log 2>&1
