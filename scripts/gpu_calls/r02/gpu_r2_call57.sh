#!/bin/bash
# replayed single-stream graphs launched straight onto the caller's stream (SVP_GRAPH_DIRECT):
# graph / async / parity tests, cfg1 / cfg2 / cfg5 A/B
o=gpurun_out/r2c57; mkdir -p $o
timeout 900 python -m pytest tests/test_gpu_f4.py tests/test_gpu_async.py tests/test_gpu_parity.py tests/test_gpu_fuzz.py -q -p no:cacheprovider -x > $o/pytest.txt 2>&1
echo "rc=$?" >> $o/pytest.txt
for i in 1 2; do
  for g in 1 0; do
    for c in 1 2; do
      SVP_GRAPH_DIRECT=$g timeout 600 python bench.py --config $c --steps 300 --warmup 20 --no-serial --no-e2e --no-cpu --no-alt > $o/cfg${c}_gd${g}_$i.json 2> $o/cfg${c}_gd${g}_$i.err
    done
  done
done
for g in 1 0; do
  SVP_GRAPH_DIRECT=$g timeout 600 python bench.py --no-serial --no-e2e --no-cpu --no-alt > $o/cfg5_gd${g}.json 2> $o/cfg5_gd${g}.err
done
