"""Max observed error of the fp32 sgemm implementations vs the oracle, in units of the
componentwise bound (|A||B|)_ij (the parity test asserts <= 1e-5).  GPU diagnostic."""
import json
import sys

import numpy as np

sys.path.insert(0, ".")
sys.path.insert(0, "tests")
import oracle  # noqa: E402
import workloads as W  # noqa: E402
from gpu_common import run_svp  # noqa: E402
from paper_conf_dac_jungc15_b200 import svp  # noqa: E402

out = {}
for name, impl in (("ffma", svp.SGEMM_FFMA), ("3xtf32", svp.SGEMM_3XTF32), ("tf32bf16", svp.SGEMM_TF32BF16)):
    res = {}
    for shape in ((512, 512, 512), (1024, 1024, 2048)):
        M, N, K = shape
        specs = [W.JobSpec(v, "sgemm", M=M, N=N, K=K) for v in range(2)]
        inputs = [W.make_inputs(s) for s in specs]
        outs, _, _ = run_svp(specs, inputs, "device", sgemm_impl=impl)
        worst, rms = 0.0, []
        for s, inp, got in zip(specs, inputs, outs):
            want = oracle.run_job(s, inp)["C"].astype(np.float64)
            A, B = inp["A"].astype(np.float64), inp["B"].astype(np.float64)
            scale = np.abs(A) @ np.abs(B)
            r = np.abs(got["C"].astype(np.float64) - want) / scale
            worst = max(worst, float(r.max()))
            rms.append(float(np.sqrt((r ** 2).mean())))
        res[f"{M}x{N}x{K}"] = {"max_err_over_bound": worst, "rms_err_over_bound": float(np.mean(rms))}
    out[name] = res
print(json.dumps(out, indent=1))
