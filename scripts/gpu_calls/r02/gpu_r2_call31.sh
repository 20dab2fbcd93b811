#!/bin/bash
# async stats test fix + full GPU suite at HEAD (graph + async defaults), smoke
o=gpurun_out/r2c31; mkdir -p $o
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > $o/pytest_gpu.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $o/smoke.txt 2>&1
for cfg in 1 2; do
  timeout 600 python bench.py --config $cfg --no-cpu --no-alt --no-serial --e2e-steps 30 --async-flush 0 > $o/e2e_cfg${cfg}_async0.json 2> /dev/null
  timeout 600 python bench.py --config $cfg --no-cpu --no-alt --no-serial --e2e-steps 30 --async-flush 1 > $o/e2e_cfg${cfg}_async1.json 2> /dev/null
done
