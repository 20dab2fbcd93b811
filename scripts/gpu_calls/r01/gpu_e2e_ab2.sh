# e2e (host-resident, PCIe) A/B: chunk cap x arena size
OUT=gpurun_out
for mc in 8 16 32; do for ag in 4 16; do
  SVP_BENCH_MAXCH=$mc timeout 900 python bench.py --steps 5 --warmup 3 --no-serial --no-alt --no-cpu --arena-gb $ag --e2e-steps 5 > $OUT/bench_e2e_mc${mc}_ag${ag}.log 2>&1
done; done
