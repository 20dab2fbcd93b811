#!/bin/bash
# final check at HEAD: the SGEMM kernel-variant tests (incl. SVP_TC_EARLY=0), smoke, the default
# bench line exactly as the driver runs it, and the reference arm
o=gpurun_out/r2c48; mkdir -p $o
python -c "import __graft_entry__ as g; g.build()" > $o/build.txt 2>&1
timeout 900 python -m pytest tests/test_gpu_sgemm_tc.py -q -p no:cacheprovider -k variants > $o/pytest_variants.txt 2>&1
echo "rc=$?" >> $o/pytest_variants.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $o/smoke.txt 2>&1
timeout 900 python bench.py --gpus 1 --steps 30 --warmup 5 > $o/bench_default.json 2> $o/bench_default.err
timeout 900 python bench.py --impl reference --gpus 1 --steps 30 --warmup 5 > $o/bench_reference.json 2> $o/bench_reference.err
