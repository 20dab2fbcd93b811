"""Margin of the default TF32+2xBF16 "sgemm" at the benched K = 2048 (DESIGN R23): relative
Frobenius error and the max componentwise ratio over several seeds and operand distributions
(U[-1,1), U[0,1) -- no cancellation, so the accumulation bias is relative to |A||B| --,
N(0,1)).  One JSON line per case."""
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

K = int(os.environ.get("ACC_K", "2048"))
KCHUNK = int(os.environ.get("ACC_KCHUNK", "0"))  # svp_config.sgemm_kchunk (strict mode, R23)
MN = 512
for dist in ("u11", "u01", "normal"):
    for seed in range(4):
        g = np.random.default_rng(100 + seed)
        specs = [W.JobSpec(v, "sgemm", M=MN, N=MN, K=K) for v in range(2)]
        if dist == "u11":
            mk = lambda *s: (g.random(s, dtype=np.float32) * 2 - 1).astype(np.float32)
        elif dist == "u01":
            mk = lambda *s: g.random(s, dtype=np.float32)
        else:
            mk = lambda *s: g.standard_normal(s, dtype=np.float32)
        inputs = [{"A": mk(MN, K), "B": mk(K, MN)} for _ in specs]
        want = oracle.run_jobs(specs, inputs, threads=2)
        for name, impl in (("tf32bf16", svp.SGEMM_TF32BF16), ("ffma", svp.SGEMM_FFMA)):
            outs, _, _ = run_svp(specs, inputs, "device", sgemm_impl=impl, sgemm_kchunk=KCHUNK)
            for i in range(2):
                G = outs[i]["C"].astype(np.float64)
                O = want[i]["C"].astype(np.float64)
                A, B = inputs[i]["A"].astype(np.float64), inputs[i]["B"].astype(np.float64)
                d = G - O
                print(json.dumps({"impl": name, "dist": dist, "seed": seed, "vp": i, "K": K, "kchunk": KCHUNK,
                                  "frob_rel": float(np.linalg.norm(d) / np.linalg.norm(O)),
                                  "bias_beta": float((d * O).sum() / (O * O).sum()),
                                  "max_comp_ratio": float((np.abs(d) / (np.abs(A) @ np.abs(B))).max())}), flush=True)
