"""Where does cfg5's interleaved step lose time?  Times the SGEMM-only and memory-bound-only
subsets of config 5 and the full mix (interleaved / one stream / co-scheduled), each for a
bench-length window (~30 steps) and a long window (~2 s) with nvidia-smi power + SM clock
sampled during the long one.  Writes gpurun_out/overlap_probe.json."""
import json
import os
import subprocess
import sys
import tempfile
import time

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import workloads as W  # noqa: E402
from paper_conf_dac_jungc15_b200 import svp  # noqa: E402
from paper_conf_dac_jungc15_b200.vpset import VPSet  # noqa: E402


def sample_start():
    f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
    p = subprocess.Popen(["nvidia-smi", "--id=0", "--query-gpu=power.draw,clocks.sm,clocks_event_reasons.sw_power_cap",
                          "--format=csv,noheader,nounits", "-lms", "50"], stdout=f, stderr=subprocess.DEVNULL)
    time.sleep(0.3)
    return f, p


def sample_stop(f, p):
    p.terminate()
    p.wait()
    f.seek(0)
    rows = []
    for line in f.read().splitlines():
        x = [t.strip() for t in line.split(",")]
        try:
            rows.append((float(x[0]), float(x[1]), x[2]))
        except (ValueError, IndexError):
            pass
    rows = rows[4:] if len(rows) > 8 else rows
    if not rows:
        return {}
    pw = sorted(r[0] for r in rows)
    ck = sorted(r[1] for r in rows)
    return {"power_w_median": pw[len(pw) // 2], "sm_mhz_median": ck[len(ck) // 2],
            "power_cap_frac": sum(1 for r in rows if r[2].lower().startswith("active")) / len(rows), "samples": len(rows)}


def run(name, specs, inputs, steps_short=30, long_s=2.0, **kw):
    ctx = svp.Context(num_gpus=1, device_ids=[0], **kw)
    vs = VPSet(ctx, specs, inputs, "device")
    jb = svp.JobBatch(vs.job_list())
    for _ in range(3):
        ctx.submit_batch(jb)
        ctx.flush()
    torch.cuda.synchronize()
    # short window (bench-like), after an idle gap so the power state starts cool
    time.sleep(1.0)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(steps_short):
        ctx.submit_batch(jb)
        ctx.flush()
    e1.record()
    torch.cuda.synchronize()
    short_ms = e0.elapsed_time(e1) / steps_short
    f, p = sample_start()
    n = 0
    t0 = time.time()
    e0.record()
    while time.time() - t0 < long_s:
        ctx.submit_batch(jb)
        ctx.flush()
        n += 1
    e1.record()
    torch.cuda.synchronize()
    long_ms = e0.elapsed_time(e1) / n
    pw = sample_stop(f, p)
    ctx.close()
    del vs
    r = {"jobs": len(specs), "short_ms_per_step": short_ms, "long_ms_per_step": long_ms, **pw}
    print(name, json.dumps(r), flush=True)
    return r


def main():
    torch.cuda.set_device(0)
    specs = W.config_specs(5)
    inputs = W.make_inputs_many(specs)
    sg = [i for i, s in enumerate(specs) if s.kernel == "sgemm"]
    mb = [i for i, s in enumerate(specs) if s.kernel != "sgemm"]
    pick = lambda idx: ([specs[i] for i in idx], [inputs[i] for i in idx])  # noqa: E731
    res = {}
    res["sgemm_only"] = run("sgemm_only", *pick(sg))
    res["membound_only"] = run("membound_only", *pick(mb))
    for k in ("vecadd", "saxpy", "hist256", "blackscholes"):
        idx = [i for i, s in enumerate(specs) if s.kernel == k]
        res[k + "_only"] = run(k + "_only", *pick(idx))
    res["all_interleaved"] = run("all_interleaved", specs, inputs)
    res["all_one_stream"] = run("all_one_stream", specs, inputs, interleave=False)
    os.environ["SVP_COSCHEDULE"] = "1"
    res["all_coschedule"] = run("all_coschedule", specs, inputs)
    os.environ.pop("SVP_COSCHEDULE")
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    with open(os.path.join(ROOT, "gpurun_out", "overlap_probe.json"), "w") as f:
        json.dump(res, f, indent=1)


if __name__ == "__main__":
    main()
