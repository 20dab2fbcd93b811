#!/bin/bash
# Fig 9(a) on B200: kernel-length sweep of two interleaved programs (tools/sweeps.py S3a)
mkdir -p gpurun_out/r2c22
timeout 1200 python tools/sweeps.py --only a --out gpurun_out/r2c22/s3a.json > gpurun_out/r2c22/s3a.log 2>&1
