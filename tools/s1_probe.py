"""S1 probe: where does the time of a coalesced vecadd flush go as the constant total of
2^26 elements is split over more VPs (Fig 10a)?  Prints, per N, the
event-timed submit+flush, the host plan / issue / total of the flush, and the kernel's own
event-timed duration (profile_level 1), for the global and the by-value segment table and
the validate_ptrs levels 1 (allocation ranges remembered), 2 (queried per submit) and 0."""
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


def run(N, table_mode, validate):
    total = 1 << 26
    specs = [W.JobSpec(v, "vecadd", n=total // N) for v in range(N)]
    c = svp.Context(num_gpus=1, external_streams=[torch.cuda.current_stream().cuda_stream], profile_level=1,
                    table_mode=table_mode, validate_ptrs=validate)
    vs = VPSet(c, specs, [W.make_inputs(s) for s in specs], "device")
    jobs = svp.JobBatch(vs.job_list())
    s = torch.cuda.current_stream()
    for _ in range(3):
        c.submit_batch(jobs)
        c.flush()
    ts, fs = [], []
    c.reset_profile()
    for _ in range(7):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record(s)
        c.submit_batch(jobs)
        c.flush()
        e1.record(s)
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
        fs.append(c.flush_stats())
    ks = c.kernel_stats(c.kernel_ids["vecadd"])
    row = {"N": N, "table_mode": table_mode, "validate": validate, "flush_ms": statistics.median(ts),
           "kernel_ms": ks["total_ns"] / ks["launches"] / 1e6, "launches": ks["launches"] / 7,
           "host_plan_us": statistics.median(f["host_plan_ns"] / 1e3 for f in fs) if "host_plan_ns" in fs[0] else None,
           "stats": {k: v for k, v in fs[-1].items()}}
    c.close()
    del vs
    torch.cuda.empty_cache()
    return row


if __name__ == "__main__":
    for N in (1, 16, 64, 128, 240, 256):
        for tm in (0, 1):
            for val in (1, 2, 0):
                print(json.dumps(run(N, tm, val)), flush=True)
