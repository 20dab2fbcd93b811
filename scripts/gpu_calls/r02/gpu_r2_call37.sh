#!/bin/bash
# final-state measurement pass at HEAD: GPU suite, smoke, bench lines for BASELINE configs 1-5
# (full lines: serial baselines, e2e, oracle), reference arm, 2 logical GPUs, ncu launch list
# and --set full of the SGEMM and hist256 launches
o=gpurun_out/r2c37; mkdir -p $o
python -c "import __graft_entry__ as g; g.build()" > $o/build.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > $o/pytest_gpu.txt 2>&1
echo "rc=$?" >> $o/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $o/smoke.txt 2>&1
timeout 900 python bench.py > $o/bench_cfg5.json 2> $o/bench_cfg5.err
for c in 1 2 3 4; do
  timeout 900 python bench.py --config $c > $o/bench_cfg$c.json 2> $o/bench_cfg$c.err
done
timeout 900 python bench.py --impl reference > $o/bench_reference_cfg5.json 2> $o/bench_reference_cfg5.err
SVP_BENCH_DEVICES=0,0 timeout 900 python bench.py --gpus 2 --no-serial --no-cpu --no-e2e > $o/bench_cfg5_gpus2_logical.json 2> $o/bench_cfg5_gpus2_logical.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $o/launches.csv \
    python bench.py --steps 2 --warmup 3 --no-serial --no-alt --no-e2e --no-cpu > $o/launches_bench.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_sgemm_tc -s 2 -c 1 -o $o/sgemm_full \
    python bench.py --steps 1 --warmup 3 --no-serial --no-alt --no-e2e --no-cpu > $o/sgemm_full.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_hist256 -s 2 -c 1 -o $o/hist_full \
    python bench.py --steps 1 --warmup 3 --no-serial --no-alt --no-e2e --no-cpu > $o/hist_full.log 2>&1
ls -la $o
