"""Probe: do the K-chunk folds keep subnormal partial sums?  (GPU, A/B of the epilogue.)

Two VPs of SGEMM 512 x 256 x 2048 (K > the 768-k chunk, beta = 0) with A ~ 2^-64 U[1,2),
B ~ 2^-74 U[1,2): products ~2^-138, one chunk's partial ~2^-129 (subnormal), C ~2^-127.
Prints, per output, the max |g - o| in units of 2^-149 and how many outputs differ from the
oracle by more than (K + 1) 2^-149 (the tolerance the IEEE test allows for subnormal
accumulation).  Run once per epilogue (SVP_TC_EPI=0 TMA reduce-add, =1 red.global.add).
"""
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.join(os.path.dirname(__file__), "..", "tests"))
sys.path.insert(0, os.path.join(os.path.dirname(__file__), ".."))

import oracle  # noqa: E402
import workloads as W  # noqa: E402
from gpu_common import run_svp  # noqa: E402


def main():
    M, N, K = 512, 256, 2048
    g = np.random.default_rng(5)
    specs = [W.JobSpec(v, "sgemm", M=M, N=N, K=K) for v in range(2)]
    inputs = []
    for _ in specs:
        A = (np.float32(2.0 ** -64) * (1 + g.random((M, K), dtype=np.float32))).astype(np.float32)
        B = (np.float32(2.0 ** -74) * (1 + g.random((K, N), dtype=np.float32))).astype(np.float32)
        inputs.append({"A": A, "B": B, "C": np.zeros((M, N), np.float32)})
    outs, _, _ = run_svp(specs, inputs, "device")
    res = []
    for s, inp, got in zip(specs, inputs, outs):
        O = oracle.sgemm(inp["A"], inp["B"], None, 1.0, 0.0).astype(np.float64)
        G = got["C"].astype(np.float64)
        err = np.abs(G - O) / 2.0 ** -149
        res.append({"vp": s.vp, "max_err_ulp149": float(err.max()), "median_out_log2": float(np.log2(np.median(O))),
                    "over_tol": int((err > K + 1).sum()), "rel_max": float((np.abs(G - O) / O).max())})
    print(json.dumps({"epi": os.environ.get("SVP_TC_EPI", "0"), "stagger": os.environ.get("SVP_TC_STAGGER", "0"),
                      "res": res}))


if __name__ == "__main__":
    main()
