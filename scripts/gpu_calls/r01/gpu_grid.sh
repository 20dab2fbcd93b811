OUT=gpurun_out; : > $OUT/grid.jsonl
for cfg in "8 4" "4 4" "2 2" "1 1" "2 4" "4 2"; do set -- $cfg
  SVP_EW_PER_SM=$1 SVP_BS_PER_SM=$2 timeout 300 python tools/grid_probe.py vecadd,blackscholes,membound,all 2>&1 | grep RESULT | sed 's/^RESULT //' >> $OUT/grid.jsonl
done
python -c "
import json
for l in open('$OUT/grid.jsonl'):
    d=json.loads(l); print(d['subset'], d['ew_per_sm'], d['bs_per_sm'], round(d['short_ms_per_step'],3), round(d['long_ms_per_step'],3), d.get('power_w_median'), d.get('sm_mhz_median'))
"
