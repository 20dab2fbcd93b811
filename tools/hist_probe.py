"""hist256 balance probe: event-timed coalesced hist256 launches over 8 VPs of 16 Mi bytes
with uniform, 90 %-one-value (the cfg3-5 skewed variant) and constant data, and the cfg5
hist256 subset, so per-byte cost by distribution (and the cfg5 launch) can be compared."""
import json
import os
import statistics
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import workloads as W  # noqa: E402
from paper_conf_dac_jungc15_b200 import svp  # noqa: E402
from paper_conf_dac_jungc15_b200.vpset import VPSet  # noqa: E402


def timed(specs, inputs, reps=9):
    c = svp.Context(num_gpus=1, external_streams=[torch.cuda.current_stream().cuda_stream], profile_level=1)
    vs = VPSet(c, specs, inputs, "device")
    jb = svp.JobBatch(vs.job_list())
    for _ in range(3):
        c.submit_batch(jb)
        c.flush()
    c.reset_profile()
    for _ in range(reps):
        c.submit_batch(jb)
        c.flush()
    ks = c.kernel_stats(c.kernel_ids["hist256"])
    ms = ks["total_ns"] / ks["launches"] / 1e6
    nbytes = sum(s.n for s in specs)
    c.close()
    del vs
    torch.cuda.empty_cache()
    return {"ms": ms, "bytes": nbytes, "tbs": nbytes / ms / 1e9}


if __name__ == "__main__":
    n = 1 << 24
    out = {}
    for name in ("uniform", "skew90", "constant"):
        specs = [W.JobSpec(v, "hist256", n=n, skew=(name == "skew90")) for v in range(8)]
        inputs = [W.make_inputs(s) for s in specs]
        if name == "constant":
            for inp in inputs:
                inp["d"][:] = 7
        out[name] = timed(specs, inputs)
        print(name, json.dumps(out[name]), flush=True)
    specs = [s for s in W.config_specs(5) if s.kernel == "hist256"]
    out["cfg5_hist"] = timed(specs, W.make_inputs_many(specs))
    print("cfg5_hist", json.dumps(out["cfg5_hist"]), flush=True)
    if len(sys.argv) > 1:
        json.dump(out, open(sys.argv[1], "w"), indent=1)
