#!/bin/bash
# pipelined flushes: async tests + parity/f4 regression, then bench cfg1/cfg2/cfg5 with --async-flush 0/1
o=gpurun_out/r2c30; mkdir -p $o
timeout 900 python -m pytest tests/test_gpu_async.py tests/test_gpu_f4.py tests/test_gpu_parity.py tests/test_gpu_vp_control.py -q -p no:cacheprovider > $o/pytest.txt 2>&1
for i in 1 2; do
  for cfg in 1 2; do
    for a in 0 1; do
      timeout 600 python bench.py --config $cfg --no-cpu --no-alt --async-flush $a > $o/cfg${cfg}_async${a}_$i.json 2> $o/cfg${cfg}_async${a}_$i.err
    done
  done
done
for a in 0 1; do
  timeout 600 python bench.py --no-cpu --no-alt --no-serial --async-flush $a > $o/cfg5_async${a}.json 2> $o/cfg5_async${a}.err
done
