"""Host-path phase times of a launch-bound flush (S6's mix): submit, flush, plan, issue, device.

python tools/host_phases.py [--out f.json]   (GPU; runs from any checkout of this repo, so the
same script times an older tree for an A/B of the host path)
"""
import argparse
import json
import os
import statistics
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import workloads as W  # noqa: E402
from paper_conf_dac_jungc15_b200 import svp  # noqa: E402
from paper_conf_dac_jungc15_b200.vpset import VPSet  # noqa: E402


def phases(nv, reps=200, **kw):
    kinds = ("vecadd", "saxpy", "blackscholes")
    g = np.random.default_rng(nv)
    specs = [W.JobSpec(v, kinds[v % 3], n=int(g.integers(1 << 14, 1 << 16)), R=0.02, V=0.3,
                       a=float(g.uniform(-2, 2))) for v in range(nv)]
    c = svp.Context(num_gpus=1, external_streams=[torch.cuda.current_stream().cuda_stream], **kw)
    vs = VPSet(c, specs, W.make_inputs_many(specs), "device")
    jobs = svp.JobBatch(vs.job_list())
    rows = {"submit_us": [], "flush_us": [], "plan_us": [], "issue_us": [], "device_us": []}
    for r in range(reps + 10):
        t0 = time.perf_counter()
        c.submit_batch(jobs)
        t1 = time.perf_counter()
        c.flush()
        t2 = time.perf_counter()
        if r < 10:
            continue
        st = c.flush_stats()
        rows["submit_us"].append((t1 - t0) * 1e6)
        rows["flush_us"].append((t2 - t1) * 1e6)
        rows["plan_us"].append(st["host_plan_ns"] / 1e3)
        rows["issue_us"].append(st["host_issue_ns"] / 1e3)
        rows["device_us"].append(st["device_ns"] / 1e3)
    c.close()
    return {k: statistics.median(v) for k, v in rows.items()}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    torch.cuda.set_device(0)
    out = []
    for nv in (16, 256, 1024):
        for name, kw in (("default", {}), ("graph", dict(graph=True)), ("prof0", dict(profile_level=0))):
            row = {"vps": nv, "mode": name, **phases(nv, **kw)}
            print(json.dumps(row), flush=True)
            out.append(row)
    if a.out:
        with open(a.out, "w") as f:
            json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
