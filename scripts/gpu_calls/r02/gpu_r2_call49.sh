#!/bin/bash
# vecadd in dynamic tile order when alone on the GPU (SVP_VECADD_DYN): parity, cfg5 one-stream
# vecadd GB/s, cfg1 jobs/s
o=gpurun_out/r2c49; mkdir -p $o
SVP_VECADD_DYN=1 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_f4.py -q -p no:cacheprovider -x > $o/pytest_dyn.txt 2>&1
echo "rc=$?" >> $o/pytest_dyn.txt
for i in 1 2; do
  for v in 0 1; do
    SVP_VECADD_DYN=$v timeout 600 python bench.py --no-serial --no-e2e --no-cpu --no-alt > $o/cfg5_dyn${v}_$i.json 2> $o/cfg5_dyn${v}_$i.err
    SVP_VECADD_DYN=$v timeout 600 python bench.py --config 1 --steps 300 --warmup 20 --no-serial --no-e2e --no-cpu --no-alt > $o/cfg1_dyn${v}_$i.json 2> $o/cfg1_dyn${v}_$i.err
  done
done
