"""Run the Table 1 program (320^3 fp64 GEMMs) for a few levels on N VPs
(profiling target for ncu: the coalesced k_dgemm launch of one level).

    python scripts/dgemm_table1_probe.py [nvps] [iters]
"""
import os
import sys

sys.path.insert(0, os.path.join(os.path.dirname(__file__), ".."))

import torch  # noqa: E402

import workloads as W  # noqa: E402
from paper_conf_dac_jungc15_b200 import svp  # noqa: E402
from paper_conf_dac_jungc15_b200.vpset import VPSet  # noqa: E402

nv = int(sys.argv[1]) if len(sys.argv) > 1 else 8
iters = int(sys.argv[2]) if len(sys.argv) > 2 else 4
specs = W.table1_specs(nvps=nv, iters=iters)
ctx = svp.Context(num_gpus=1)
vs = VPSet(ctx, specs, [W.make_inputs(s) for s in specs], "device")
for _ in range(3):
    vs.submit()
    ctx.flush()
torch.cuda.synchronize()
st = ctx.flush_stats()
print({"vps": nv, "iters": iters, "launches": st["launches"], "levels": st["levels"]})
ctx.close()
