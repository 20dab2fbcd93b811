#!/bin/bash
# launch-bound configs after svp_flush_async: graph replay vs direct issue (cfg1, cfg2), and
# where cfg1's ~11 us of device time per step goes (ncu of its vecadd launch, launch list)
o=gpurun_out/r2c40; mkdir -p $o
for i in 1 2; do
  for c in 1 2; do
    for g in 1 0; do
      timeout 600 python bench.py --config $c --steps 200 --warmup 20 --no-serial --no-e2e --no-cpu --no-alt --graph $g > $o/cfg${c}_graph${g}_$i.json 2> $o/cfg${c}_graph${g}_$i.err
    done
  done
done
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,sm__warps_active.avg.pct_of_peak_sustained_active --clock-control none -k regex:"k_" -c 60 --csv --log-file $o/launches_cfg1.csv \
    python bench.py --config 1 --steps 20 --warmup 3 --no-serial --no-alt --no-e2e --no-cpu > $o/launches_cfg1.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_vecadd -s 30 -c 1 -o $o/vecadd_cfg1 \
    python bench.py --config 1 --steps 20 --warmup 3 --no-serial --no-alt --no-e2e --no-cpu > $o/vecadd_cfg1.log 2>&1
