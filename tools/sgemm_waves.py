"""Wave quantization of the grouped SGEMM: event-timed flushes of nv VPs x 2048^3 SGEMM
(device-resident, default TF32+2xBF16 CTA-pair kernel) for nv around cfg5's 51, so the
time per VP shows the cost of a partly filled last wave of 256x512 pair tiles
(51 VPs -> 1632 tiles over 74 pairs = 22.05 waves)."""
import json
import os
import statistics
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import workloads as W  # noqa: E402
from paper_conf_dac_jungc15_b200 import svp  # noqa: E402
from paper_conf_dac_jungc15_b200.vpset import VPSet  # noqa: E402

rows = []
for nv in [int(x) for x in (sys.argv[1:] or "44 46 48 50 51 52 54 56".split())]:
    specs = [W.JobSpec(v, "sgemm", M=2048, N=2048, K=2048) for v in range(nv)]
    c = svp.Context(num_gpus=1, external_streams=[torch.cuda.current_stream().cuda_stream], profile_level=1)
    vs = VPSet(c, specs, W.make_inputs_many(specs), "device")
    jb = svp.JobBatch(vs.job_list())
    for _ in range(3):
        c.submit_batch(jb)
        c.flush()
    c.reset_profile()
    for _ in range(7):
        c.submit_batch(jb)
        c.flush()
    ks = c.kernel_stats(c.kernel_ids["sgemm"])
    ms = ks["total_ns"] / ks["launches"] / 1e6
    tiles = nv * 32
    rows.append({"vps": nv, "tiles": tiles, "waves": tiles / 74, "ms": ms, "ms_per_vp": ms / nv,
                 "tflops": ks["flops"] / ks["total_ns"] / 1e3})
    print(json.dumps(rows[-1]), flush=True)
    c.close()
    del vs
    torch.cuda.empty_cache()
