#!/bin/bash
# graph default + direct issue + plan cache: full GPU suite, smoke, bench lines cfg1-5 at the defaults, S6
o=gpurun_out/r2c27; mkdir -p $o
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > $o/pytest_gpu.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $o/smoke.txt 2>&1
timeout 900 python bench.py > $o/bench_cfg5.json 2> $o/bench_cfg5.err
for cfg in 1 2 3 4; do
  timeout 900 python bench.py --config $cfg > $o/bench_cfg$cfg.json 2> $o/bench_cfg$cfg.err
done
timeout 600 python tools/sweeps.py --only 6 --out $o/s6.json > $o/s6.log 2>&1
