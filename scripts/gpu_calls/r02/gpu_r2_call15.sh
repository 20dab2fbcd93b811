#!/bin/bash
# round 2, call 15: default kchunk 768 -- GPU suite + smoke + cfg5 bench (default) + logical 2-GPU
mkdir -p gpurun_out/r2c15
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/r2c15/pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/r2c15/pytest_gpu.txt
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r2c15/smoke.log 2>&1
python bench.py > gpurun_out/r2c15/bench_cfg5.json 2> gpurun_out/r2c15/bench_cfg5.err
SVP_BENCH_DEVICES=0,0 timeout 900 python bench.py --gpus 2 --steps 10 --warmup 3 --no-serial --no-alt --no-cpu > gpurun_out/r2c15/bench_gpus2_logical.json 2> gpurun_out/r2c15/bench_gpus2_logical.err
