#!/bin/bash
# NUMA placement (ABI 6): topology probe, GPU suite, e2e A/B host_numa 1 vs 0, Fig 9(a) sweep
o=gpurun_out/r2c23; mkdir -p $o
{ nproc; lscpu | grep -iE "socket|numa|model name"; for d in /sys/bus/pci/devices/*; do
  if [ "$(cat $d/vendor 2>/dev/null)" = "0x10de" ] && [ "$(cat $d/class 2>/dev/null | cut -c1-6)" = "0x0302" ]; then
    echo "$d node=$(cat $d/numa_node) cpus=$(cat $d/local_cpulist)"; fi; done;
  python -c "import torch;p=torch.cuda.get_device_properties(0);print('gpu0 pci',p.pci_domain_id,p.pci_bus_id,p.pci_device_id)";
  python -c "import os;print('affinity',len(os.sched_getaffinity(0)))"; } > $o/topology.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > $o/pytest_gpu.txt 2>&1
for i in 1 2; do
  for n in 1 0; do
    timeout 600 python bench.py --steps 10 --warmup 3 --no-serial --no-alt --no-cpu --host-numa $n --e2e-steps 5 > $o/bench_numa${n}_$i.json 2> $o/bench_numa${n}_$i.err
  done
done
timeout 1200 python tools/sweeps.py --only a --out $o/s3a.json > $o/s3a.log 2>&1
