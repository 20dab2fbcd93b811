"""Run the cfg5 SGEMM group (51 x 2048^3) back to back for ~3 s per implementation and
sample power / SM clock with nvidia-smi (is the tensor-core SGEMM power-bound?)."""
import json
import subprocess
import sys
import tempfile
import time

import torch

sys.path.insert(0, ".")
import workloads as W  # noqa: E402
from paper_conf_dac_jungc15_b200 import svp  # noqa: E402
from paper_conf_dac_jungc15_b200.vpset import VPSet  # noqa: E402

specs = [s for s in W.config_specs(5) if s.kernel == "sgemm"]
inputs = W.make_inputs_many(specs)
res = {}
for name, impl in (("tf32bf16", svp.SGEMM_TF32BF16), ("3xtf32", svp.SGEMM_3XTF32), ("ffma", svp.SGEMM_FFMA)):
    ctx = svp.Context(num_gpus=1, sgemm_impl=impl, graph=True)
    vs = VPSet(ctx, specs, inputs, "device")
    jb = svp.JobBatch(vs.job_list())
    for _ in range(3):
        ctx.submit_batch(jb)
        ctx.flush()
    f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
    p = subprocess.Popen(["nvidia-smi", "--id=0", "--query-gpu=power.draw,clocks.sm,power.limit",
                          "--format=csv,noheader,nounits", "-lms", "100"], stdout=f)
    t0 = time.time()
    n = 0
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    while time.time() - t0 < 3.0:
        ctx.submit_batch(jb)
        ctx.flush()
        n += 1
    e1.record()
    torch.cuda.synchronize()
    p.terminate()
    p.wait()
    f.seek(0)
    rows = [[float(x) for x in l.split(",")] for l in f.read().splitlines() if l.strip()]
    rows = rows[3:]  # drop ramp-up
    ms = e0.elapsed_time(e1) / n
    tf = sum(2.0 * s.M * s.N * s.K for s in specs) / (ms / 1e3) / 1e12
    res[name] = {"ms_per_launch": ms, "tflops": tf, "power_w_median": sorted(r[0] for r in rows)[len(rows) // 2],
                 "power_w_max": max(r[0] for r in rows), "sm_mhz_median": sorted(r[1] for r in rows)[len(rows) // 2],
                 "power_limit_w": rows[0][2], "samples": len(rows)}
    ctx.close()
    del vs
    torch.cuda.empty_cache()
print(json.dumps(res, indent=1))
