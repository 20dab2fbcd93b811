#!/bin/bash
# re-entry: full GPU suite + smoke + cfg5 default bench at HEAD (graph + async defaults)
o=gpurun_out/r2c33; mkdir -p $o
python -c "import __graft_entry__ as g; g.build()" > $o/build.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > $o/pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> $o/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $o/smoke.txt 2>&1
timeout 900 python bench.py > $o/bench_cfg5.json 2> $o/bench_cfg5.err
