#!/bin/bash
# round 2, call 7: mode-H (host-resident) timeline diagnostics
mkdir -p gpurun_out/r2c7
python tools/e2e_timeline.py --out gpurun_out/r2c7/tl_default.json > gpurun_out/r2c7/tl.log 2>&1
CUDA_DEVICE_MAX_CONNECTIONS=32 python tools/e2e_timeline.py --out gpurun_out/r2c7/tl_conn32.json >> gpurun_out/r2c7/tl.log 2>&1
python tools/e2e_timeline.py --streams 2 --out gpurun_out/r2c7/tl_s2.json >> gpurun_out/r2c7/tl.log 2>&1
python tools/e2e_timeline.py --profile 0 >> gpurun_out/r2c7/tl.log 2>&1
CUDA_DEVICE_MAX_CONNECTIONS=32 python tools/e2e_timeline.py --profile 0 >> gpurun_out/r2c7/tl.log 2>&1
