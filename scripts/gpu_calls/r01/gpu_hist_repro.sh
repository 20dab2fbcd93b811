OUT=gpurun_out
r() { name=$1; shift; timeout 300 env "$@" > $OUT/hr_$name.log 2>&1; echo "$name: $(tail -1 $OUT/hr_$name.log)"; }
r wide_all SVP_TC_WIDE=1 python scripts/hist_repro.py 16 all
r wide_all2 SVP_TC_WIDE=1 python scripts/hist_repro.py 16 all
r pair_all SVP_TC_WIDE=0 python scripts/hist_repro.py 16 all
