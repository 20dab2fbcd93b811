# e2e (host-resident, PCIe-bound) A/B: staging arena size and chunk count
OUT=gpurun_out
for cfg in "8 8" "16 8" "24 8" "24 16" "24 4"; do
  set -- $cfg
  SVP_BENCH_MAXCH=$2 timeout 600 python bench.py --steps 3 --warmup 3 --no-serial --no-cpu --no-alt --arena-gb $1 --e2e-steps 5 > $OUT/e2e_a$1_c$2.log 2>&1
  tail -1 $OUT/e2e_a$1_c$2.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); e=d['e2e']; print('arena $1 chunks $2', round(e['value']), round(e['ms_per_step'],1), e['chunks'])"
done
