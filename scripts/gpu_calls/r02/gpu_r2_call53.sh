#!/bin/bash
# final full GPU suite + smoke + default bench at HEAD (after the split-K DGEMM)
o=gpurun_out/r2c53; mkdir -p $o
python -c "import __graft_entry__ as g; g.build()" > $o/build.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > $o/pytest_gpu.txt 2>&1
echo "rc=$?" >> $o/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $o/smoke.txt 2>&1
timeout 900 python bench.py > $o/bench_default.json 2> $o/bench_default.err
