"""Repro for a cfg5 hist256 mismatch: run the bench's cfg5 launch configuration for several
steps and, after each, compare every hist VP's counts with np.bincount of the host input,
and the device copy of the input with the host input (argv[1] = steps)."""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import workloads as W  # noqa: E402
from paper_conf_dac_jungc15_b200 import svp  # noqa: E402
from paper_conf_dac_jungc15_b200.vpset import VPSet  # noqa: E402

steps = int(sys.argv[1]) if len(sys.argv) > 1 else 6
only = sys.argv[2] if len(sys.argv) > 2 else "all"
specs = W.config_specs(5)
if only == "nosgemm":
    specs = [s for s in specs if s.kernel != "sgemm"]
elif only == "histsgemm":
    specs = [s for s in specs if s.kernel in ("sgemm", "hist256")]
inputs = W.make_inputs_many(specs)
stream = torch.cuda.current_stream()
import os  # noqa: E402
ctx = svp.Context(num_gpus=1, device_ids=[0], profile_level=1, external_streams=[stream.cuda_stream],
                  validate_ptrs=True, sgemm_impl=int(os.environ.get("REPRO_IMPL", svp.SGEMM_TF32BF16)),
                  table_mode=int(os.environ.get("REPRO_TABLE", svp.TABLE_PARAM)),
                  interleave=bool(int(os.environ.get("REPRO_INTERLEAVE", "1"))))
vs = VPSet(ctx, specs, inputs, "device", device_ordinals=[0])
jobs = svp.JobBatch(vs.job_list())
hist = [i for i, s in enumerate(specs) if s.kernel == "hist256"]
want = {i: np.bincount(inputs[i]["d"], minlength=256).astype(np.uint32) for i in hist}
bad_total = 0
for step in range(steps):
    ctx.submit_batch(jobs)
    ctx.flush()
    torch.cuda.synchronize()
    for i in hist:
        got = vs.output(i)["counts"]
        if not np.array_equal(got, want[i]):
            bad_total += 1
            dev_d = vs.bufs[i]["d"].cpu().numpy()
            intact = np.array_equal(dev_d, inputs[i]["d"])
            diff = got.astype(np.int64) - want[i].astype(np.int64)
            print(f"step {step} vp {specs[i].vp} n {specs[i].n} misalign {specs[i].misalign} skew {specs[i].skew}: "
                  f"sum got {int(got.sum())} want {specs[i].n} |diff| {int(np.abs(diff).sum())} "
                  f"bins {int((diff != 0).sum())} input_intact {intact}", flush=True)
print(f"{only}: {bad_total} bad (vp, step) pairs over {steps} steps x {len(hist)} hist VPs; guards",
      vs.guards_intact(), flush=True)
