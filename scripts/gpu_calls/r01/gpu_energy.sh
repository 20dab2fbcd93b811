# energy per SGEMM group for every implementation (scripts/energy_probe.py)
OUT=gpurun_out/energy.jsonl; : > $OUT
nvidia-smi --query-gpu=power.draw,clocks.sm --format=csv >> gpurun_out/energy_idle.txt
run() { timeout 120 env "$@" >> $OUT 2>> gpurun_out/energy.err; }
run SVP_X=0 python scripts/energy_probe.py sgemm_tf32 2 tf32_plain_1cta
run SVP_X=0 python scripts/energy_probe.py sgemm 2 tf32bf16_pair
run SVP_TC_CTA_PAIR=0 python scripts/energy_probe.py sgemm 2 tf32bf16_1cta
run SVP_TC_TMEM_A=1 python scripts/energy_probe.py sgemm 2 tf32bf16_tmema_pair
run SVP_X=0 python scripts/energy_probe.py sgemm 1 3xtf32_pair
run SVP_TC_CTA_PAIR=0 python scripts/energy_probe.py sgemm 1 3xtf32_1cta
run SVP_X=0 python scripts/energy_probe.py sgemm 0 ffma
cat $OUT
