#!/bin/bash
# round 2, call 16: ncu evidence -- launch list of the bench command (cold, serialised) and
# --set full captures of the SGEMM (default K chunks) and hist256 launches
mkdir -p gpurun_out/r2c16
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r2c16/launches.csv \
    python bench.py --steps 2 --warmup 3 --no-serial --no-alt --no-e2e --no-cpu > gpurun_out/r2c16/launches_bench.log 2>&1
ncu --set full --import-source on --clock-control none -k regex:k_sgemm_tc -s 2 -c 1 -o gpurun_out/r2c16/sgemm_full \
    python bench.py --steps 1 --warmup 3 --no-serial --no-alt --no-e2e --no-cpu > gpurun_out/r2c16/sgemm_full.log 2>&1
ncu --set full --import-source on --clock-control none -k regex:k_hist256 -s 2 -c 1 -o gpurun_out/r2c16/hist_full \
    python bench.py --steps 1 --warmup 3 --no-serial --no-alt --no-e2e --no-cpu > gpurun_out/r2c16/hist_full.log 2>&1
SVP_SGEMM_KCHUNK_DUMMY=1 ncu --set full --import-source on --clock-control none -k regex:k_sgemm_tc -s 2 -c 1 -o gpurun_out/r2c16/sgemm_full_kc0 \
    python bench.py --steps 1 --warmup 3 --no-serial --no-alt --no-e2e --no-cpu --sgemm-kchunk 0 > gpurun_out/r2c16/sgemm_full_kc0.log 2>&1
ls -la gpurun_out/r2c16
