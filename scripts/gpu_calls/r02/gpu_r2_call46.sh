#!/bin/bash
# sweeps S1-S6 at the final HEAD (S6 now with pipelined rounds), then the full GPU suite and smoke
o=gpurun_out/r2c46; mkdir -p $o
timeout 1800 python tools/sweeps.py --out $o/sweeps_final_s3.json > $o/sweeps.log 2>&1
echo "sweeps rc=$?" >> $o/sweeps.log
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > $o/pytest_gpu.txt 2>&1
echo "rc=$?" >> $o/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $o/smoke.txt 2>&1
