#!/bin/bash
# round 2, call 4: IEEE fix (satfinite heads only), accuracy vs K, hist scheme ceilings, GPU suite
mkdir -p gpurun_out/r2c4
python scripts/ieee_probe.py > gpurun_out/r2c4/ieee_probe.jsonl 2>/dev/null
python scripts/sgemm_accuracy_k.py > gpurun_out/r2c4/accuracy_k.jsonl 2> gpurun_out/r2c4/accuracy_k.err
python tools/hist_schemes.py --out gpurun_out/r2c4/hist_schemes.json > gpurun_out/r2c4/hist_schemes.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/r2c4/pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/r2c4/pytest_gpu.txt
