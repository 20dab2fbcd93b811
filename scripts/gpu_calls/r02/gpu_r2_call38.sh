#!/bin/bash
# cross-flush pipelining (SVP_PIPELINE=1: per-VP ordering instead of a whole-GPU barrier between
# flushes): parity/async/f4 tests under it, same-box A/B of cfg5 / cfg3 / cfg4, launch list
o=gpurun_out/r2c38; mkdir -p $o
SVP_PIPELINE=1 timeout 900 python -m pytest tests/test_gpu_async.py tests/test_gpu_parity.py tests/test_gpu_f4.py tests/test_gpu_vp_control.py -q -p no:cacheprovider -x > $o/pytest_pipe.txt 2>&1
echo "rc=$?" >> $o/pytest_pipe.txt
for i in 1 2; do
  for p in 0 1; do
    SVP_PIPELINE=$p timeout 600 python bench.py --steps 30 --warmup 5 --no-serial --no-e2e --no-cpu --no-alt > $o/cfg5_pipe${p}_$i.json 2> $o/cfg5_pipe${p}_$i.err
  done
  SVP_PIPELINE=0 timeout 600 python bench.py --steps 30 --warmup 5 --no-serial --no-e2e --no-cpu --no-alt --graph 0 > $o/cfg5_pipe0_graph0_$i.json 2> $o/cfg5_pipe0_graph0_$i.err
done
for c in 3 4; do
  for p in 0 1; do
    SVP_PIPELINE=$p timeout 600 python bench.py --config $c --no-serial --no-e2e --no-cpu --no-alt > $o/cfg${c}_pipe$p.json 2> $o/cfg${c}_pipe$p.err
  done
done
SVP_PIPELINE=1 timeout 600 python bench.py --steps 300 --warmup 5 --no-serial --no-e2e --no-cpu --no-alt > $o/cfg5_pipe1_300.json 2> $o/cfg5_pipe1_300.err
SVP_PIPELINE=0 timeout 600 python bench.py --steps 300 --warmup 5 --no-serial --no-e2e --no-cpu --no-alt > $o/cfg5_pipe0_300.json 2> $o/cfg5_pipe0_300.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_" -c 300 --csv --log-file $o/launches.csv \
    python bench.py --steps 2 --warmup 3 --no-serial --no-alt --no-e2e --no-cpu > $o/launches_bench.log 2>&1
