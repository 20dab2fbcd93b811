"""Energy per SGEMM group: cfg5's 51 x 2048^3 GEMMs flushed back to back for ~3 s with one
implementation (argv: kernel impl label), nvidia-smi power / SM clock at 50 ms.  Prints one
JSON line: ms per launch, TFLOP/s, median power, joules per launch.  Env knobs
(SVP_TC_CTA_PAIR, SVP_TC_TMEM_A) are read once per process, so each variant runs in its
own process (scripts/gpu_energy.sh)."""
import dataclasses
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

kernel, impl, label = sys.argv[1], int(sys.argv[2]), sys.argv[3]
specs = [dataclasses.replace(s, kernel=kernel) for s in W.config_specs(5) if s.kernel == "sgemm"]
inputs = W.make_inputs_many(specs)
ctx = svp.Context(num_gpus=1, sgemm_impl=impl, graph=True)
vs = VPSet(ctx, specs, inputs, "device")
jb = svp.JobBatch(vs.job_list())
for _ in range(3):
    ctx.submit_batch(jb)
    ctx.flush()
torch.cuda.synchronize()
time.sleep(1.0)
f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
p = subprocess.Popen(["nvidia-smi", "--id=0", "--query-gpu=power.draw,clocks.sm", "--format=csv,noheader,nounits",
                      "-lms", "50"], stdout=f, stderr=subprocess.DEVNULL)
time.sleep(0.3)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
n = 0
t0 = time.time()
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
rows = [[float(x) for x in l.split(",")] for l in f.read().splitlines() if l.strip()][6:]
ms = e0.elapsed_time(e1) / n
pw = sorted(r[0] for r in rows)[len(rows) // 2]
ck = sorted(r[1] for r in rows)[len(rows) // 2]
tf = sum(2.0 * s.M * s.N * s.K for s in specs) / (ms / 1e3) / 1e12
print(json.dumps({"label": label, "ms_per_launch": ms, "tflops": tf, "power_w": pw, "sm_mhz": ck,
                  "joules_per_launch": pw * ms / 1e3, "launches": n}), flush=True)
