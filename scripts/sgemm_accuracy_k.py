"""How the fp32 "sgemm" implementations' error grows with K (random U[-1,1) operands):
relative Frobenius error ||G - O||_F / ||O||_F, its projection on O (a systematic scale
bias beta with G ~ (1 + beta) O), and the max componentwise |g - o| / (|A||B|)_ij.
Prints one JSON line per (impl, K)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path[:0] = [ROOT, os.path.join(ROOT, "tests")]

import numpy as np  # noqa: E402

import oracle  # noqa: E402
import workloads as W  # noqa: E402
from gpu_common import run_svp  # noqa: E402
from paper_conf_dac_jungc15_b200 import svp  # noqa: E402

MN = int(os.environ.get("ACC_MN", "512"))
KCHUNK = int(os.environ.get("ACC_KCHUNK", "0"))  # svp_config.sgemm_kchunk (strict mode, R23)
for K in (256, 1024, 2048, 4096, 8192):
    specs = [W.JobSpec(v, "sgemm", M=MN, N=MN, K=K) for v in range(2)]
    inputs = [W.make_inputs(s) for s in specs]
    want = oracle.run_jobs(specs, inputs, threads=2)
    for name, impl in (("ffma", svp.SGEMM_FFMA), ("3xtf32", svp.SGEMM_3XTF32), ("tf32bf16", svp.SGEMM_TF32BF16)):
        outs, _, _ = run_svp(specs, inputs, "device", sgemm_impl=impl, sgemm_kchunk=KCHUNK)
        G = outs[0]["C"].astype(np.float64)
        O = want[0]["C"].astype(np.float64)
        A, B = inputs[0]["A"].astype(np.float64), inputs[0]["B"].astype(np.float64)
        d = G - O
        scale = np.abs(A) @ np.abs(B)
        print(json.dumps({"impl": name, "M": MN, "N": MN, "K": K, "kchunk": KCHUNK,
                          "frob_rel": float(np.linalg.norm(d) / np.linalg.norm(O)),
                          "bias_beta": float((d * O).sum() / (O * O).sum()),
                          "max_comp_ratio": float((np.abs(d) / scale).max())}), flush=True)
