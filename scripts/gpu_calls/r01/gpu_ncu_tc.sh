# ncu --set full of one k_sgemm_tc launch for the given impl (default tf32bf16)
IMPL=${1:-tf32bf16}
OUT=gpurun_out
mkdir -p $OUT
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_sgemm_tc" -s 1 -c 1 -o $OUT/prof_tc_$IMPL -f \
  python bench.py --steps 2 --warmup 3 --no-serial --no-e2e --no-cpu --no-alt --sgemm-impl $IMPL > $OUT/ncu_tc_$IMPL.log 2>&1; echo "ncu rc=$?"
