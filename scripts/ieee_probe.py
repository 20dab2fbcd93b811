"""Probe: what each fp32 "sgemm" implementation returns for IEEE edge values (Inf, NaN,
near-FLT_MAX, subnormals), against the oracle.  Prints one JSON line per implementation.

    python scripts/ieee_probe.py [M N K]
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path[:0] = [ROOT, os.path.join(ROOT, "tests")]

import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import workloads as W  # noqa: E402
from ieee_cases import compare, edge_inputs  # noqa: E402
from paper_conf_dac_jungc15_b200 import svp  # noqa: E402
from paper_conf_dac_jungc15_b200.vpset import VPSet  # noqa: E402

M, N, K = (int(x) for x in sys.argv[1:4]) if len(sys.argv) >= 4 else (256, 256, 64)
for kernel, impl, name in (("sgemm", svp.SGEMM_FFMA, "ffma"), ("sgemm", svp.SGEMM_3XTF32, "3xtf32"),
                           ("sgemm", svp.SGEMM_TF32BF16, "tf32bf16"), ("sgemm_tf32", 0, "sgemm_tf32")):
    for beta in (0.0, 0.5):
        specs = [W.JobSpec(v, kernel, M=M, N=N, K=K, alpha=1.0, beta=beta) for v in range(2)]
        inputs = [edge_inputs(M, N, K, seed=11 + v, beta=beta) for v in range(2)]
        ctx = svp.Context(num_gpus=1, sgemm_impl=impl)
        vs = VPSet(ctx, specs, inputs, "device")
        vs.submit()
        ctx.flush()
        torch.cuda.synchronize()
        for i, (s, inp) in enumerate(zip(specs, inputs)):
            G = vs.output(i)["C"]
            O = oracle.sgemm(inp["A"], inp["B"], inp.get("C"), s.alpha, s.beta)
            r = compare(G, O, inp["A"], inp["B"], s.alpha, s.beta, inp.get("C"), tiny_coef=0.0)
            r1 = compare(G, O, inp["A"], inp["B"], s.alpha, s.beta, inp.get("C"), tiny_coef=1.0)
            r["over_bound_tiny_coef1"] = r1["over_bound"]
            r["max_err_over_bound_tiny_coef1"] = r1["max_err_over_bound"]
            # per-row view of the subnormal rows / cols
            d = np.abs(G.astype(np.float64) - O.astype(np.float64))
            r["row10_maxerr"] = float(np.nanmax(d[10, 13:]))
            r["row11_col11"] = (float(G[11, 11]), float(O[11, 11]))
            r["row12_col12"] = (float(G[12, 12]), float(O[12, 12]))
            r["row6_maxrel"] = float(np.nanmax(d[6, 13:] / np.maximum(np.abs(O[6, 13:].astype(np.float64)), 1e-30)))
            print(json.dumps({"impl": name, "beta": beta, "vp": i, "M": M, "N": N, "K": K, **r}), flush=True)
        assert vs.guards_intact()
        ctx.close()
