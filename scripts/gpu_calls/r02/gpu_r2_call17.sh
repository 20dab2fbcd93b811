#!/bin/bash
# round 2, call 17: bench lines for BASELINE configs 1-5 at the final defaults; mode-H timeline;
# IEEE probe; Black-Scholes error report
mkdir -p gpurun_out/r2c17
python bench.py > gpurun_out/r2c17/bench_cfg5.json 2> gpurun_out/r2c17/bench_cfg5.err
for c in 1 2 3 4; do
  python bench.py --config $c > gpurun_out/r2c17/bench_cfg$c.json 2> gpurun_out/r2c17/bench_cfg$c.err
done
python bench.py --impl reference > gpurun_out/r2c17/bench_reference_cfg5.json 2> gpurun_out/r2c17/bench_reference_cfg5.err
python tools/e2e_timeline.py --out gpurun_out/r2c17/tl_default.json > gpurun_out/r2c17/tl.log 2>&1
python scripts/ieee_probe.py > gpurun_out/r2c17/ieee_probe.jsonl 2>/dev/null
python scripts/bs_error.py --out gpurun_out/r2c17/bs_error.json > gpurun_out/r2c17/bs_error.log 2>&1
