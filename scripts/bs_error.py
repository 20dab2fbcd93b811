"""Black-Scholes error report: for BASELINE cfg3's 16
Black-Scholes VPs (4 Mi options each), the coalesced sm_100a kernel against the oracle --
max |g - o| / max(|o|, S, X e^-RT) (the parity bound, must be <= 1e-5), the CUDA-SDK-style
L1 error sum|g - o| / sum|o|, and max |g - o| / |o| over options with |o| >= 1e-3 (cents).
One JSON line; --out writes it to a file too."""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path[:0] = [ROOT, os.path.join(ROOT, "tests")]

import numpy as np  # noqa: E402

import oracle  # noqa: E402
import workloads as W  # noqa: E402
from gpu_common import run_svp  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--out", default=None)
args = ap.parse_args()
specs = [s for s in W.config_specs(3) if s.kernel == "blackscholes"]
inputs = W.make_inputs_many(specs)
outs, _, _ = run_svp(specs, inputs, "device")
want = oracle.run_jobs(specs, inputs)
worst_scaled = worst_rel = 0.0
num = den = 0.0
for s, inp, got, w in zip(specs, inputs, outs, want):
    S, X, T = (inp[x].astype(np.float64) for x in "SXT")
    scale = np.maximum.reduce([np.abs(w["call"].astype(np.float64)), S, X * np.exp(-s.R * T)])
    for k in ("call", "put"):
        g, o = got[k].astype(np.float64), w[k].astype(np.float64)
        d = np.abs(g - o)
        worst_scaled = max(worst_scaled, float((d / scale).max()))
        m = np.abs(o) >= 1e-3
        worst_rel = max(worst_rel, float((d[m] / np.abs(o[m])).max()))
        num += float(d.sum())
        den += float(np.abs(o).sum())
res = {"config": "cfg3 Black-Scholes VPs", "vps": len(specs), "options": int(sum(s.n for s in specs)),
       "max_err_over_parity_scale": worst_scaled, "parity_bound": 1e-5,
       "sdk_l1_error": num / den, "max_rel_err_abs_o_ge_1e-3": worst_rel}
print(json.dumps(res))
if args.out:
    with open(args.out, "w") as f:
        json.dump(res, f, indent=1)
