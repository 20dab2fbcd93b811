#!/bin/bash
# cfg1's fixed per-launch cost: segment table by value (1-KiB kernel parameter) vs global table
o=gpurun_out/r2c51; mkdir -p $o
for i in 1 2; do
  for t in 1 0; do
    timeout 600 python bench.py --config 1 --steps 300 --warmup 20 --no-serial --no-e2e --no-cpu --no-alt --table-mode $t > $o/cfg1_table${t}_$i.json 2> $o/cfg1_table${t}_$i.err
  done
done
for t in 1 0; do
  timeout 600 ncu --metrics gpu__time_duration.sum,sm__cycles_active.avg,smsp__warps_launched.sum --clock-control none -k regex:"k_vecadd" -c 40 --csv --log-file $o/ncu_cfg1_table$t.csv \
    python bench.py --config 1 --steps 20 --warmup 3 --no-serial --no-alt --no-e2e --no-cpu --table-mode $t > $o/ncu_cfg1_table$t.log 2>&1
done
