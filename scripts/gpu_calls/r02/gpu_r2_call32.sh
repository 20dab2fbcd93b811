#!/bin/bash
# kernel_launches stat after the issue half (tail-split tests), async tests, cfg5 default line
o=gpurun_out/r2c32; mkdir -p $o
timeout 900 python -m pytest tests/test_gpu_sgemm_tc.py tests/test_gpu_async.py -q -p no:cacheprovider > $o/pytest.txt 2>&1
timeout 900 python bench.py > $o/bench_cfg5.json 2> $o/bench_cfg5.err
