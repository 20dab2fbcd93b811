"""Shared helpers for the -m gpu tests: run jobs through libsvp, compare with the oracle.

Tolerances:
  vecadd, SAXPY, hist256 -- bit-exact;
  Black-Scholes          -- |g - o| <= 1e-5 * max(|o|, S, X e^{-RT}) per option;
  SGEMM fp32             -- |g - o| <= 1e-5 * (|A||B| + |beta C|)_ij per element and
                            ||G - O||_F <= 1e-5 ||O||_F; integer inputs -> bit-exact.
"""
from __future__ import annotations

import numpy as np
import torch

import oracle
import workloads as W
from paper_conf_dac_jungc15_b200 import svp
from paper_conf_dac_jungc15_b200.vpset import VPSet

BS_TOL = 1e-5
SGEMM_TOL = 1e-5
DGEMM_TOL = 1e-12  # fp64: K * 2^-53 worst-case accumulation bound for K <= 4096 is 4.5e-13


def run_svp(specs, inputs, residency="device", **cfg):
    ctx = svp.Context(num_gpus=1, **cfg)
    try:
        vs = VPSet(ctx, specs, inputs, residency)
        vs.submit()
        ctx.flush()
        torch.cuda.synchronize()
        outs = [vs.output(i) for i in range(len(specs))]
        assert vs.guards_intact(), "a kernel wrote past a VP's buffer extent"
        prof = ctx.profile(-1)
        stats = ctx.flush_stats()
        return outs, prof, stats
    finally:
        ctx.close()


def check_job(spec, inp, got, want=None, sgemm_tol=SGEMM_TOL, sample=None):
    """Assert one job's GPU outputs match the oracle.  ``sample``: for SGEMM, a list of
    (i, j) to check one by one with oracle.sgemm_element instead of the full product."""
    k = spec.kernel
    if k in ("sgemm", "sgemm_tf32") and sample is not None:
        A, B = inp["A"], inp["B"]
        C = got["C"]
        for (i, j) in sample:
            c_old = float(inp["C"][i, j]) if spec.beta != 0 else 0.0
            o = oracle.sgemm_element(A, B, i, j, spec.alpha, spec.beta, c_old)
            scale = float(np.abs(A[i, :].astype(np.float64)) @ np.abs(B[:, j].astype(np.float64))) * abs(spec.alpha)
            scale += abs(spec.beta * c_old)
            assert abs(float(C[i, j]) - o) <= sgemm_tol * scale + 1e-30, (spec.vp, i, j, C[i, j], o)
        return
    if want is None:
        want = oracle.run_job(spec, inp)
    if k == "vecadd":
        assert np.array_equal(got["c"], want["c"]), f"vp {spec.vp} vecadd mismatch"
    elif k == "saxpy":
        assert np.array_equal(got["y"], want["y"]), f"vp {spec.vp} saxpy mismatch"
    elif k == "hist256":
        assert np.array_equal(got["counts"], want["counts"]), f"vp {spec.vp} hist mismatch"
        assert int(got["counts"].sum()) == spec.n
    elif k == "blackscholes":
        if spec.n == 0:
            return
        S, X, T = (inp[x].astype(np.float64) for x in "SXT")
        scale = np.maximum.reduce([np.abs(want["call"].astype(np.float64)), S, X * np.exp(-spec.R * T)])
        for name in ("call", "put"):
            err = np.abs(got[name].astype(np.float64) - want[name].astype(np.float64))
            bad = err > BS_TOL * scale
            assert not bad.any(), (spec.vp, name, int(bad.sum()), float((err / scale).max()))
    elif k in ("sgemm", "sgemm_tf32", "dgemm"):
        if k == "dgemm":
            sgemm_tol = DGEMM_TOL
        G, O = got["C"].astype(np.float64), want["C"].astype(np.float64)
        if spec.M * spec.N == 0:
            return
        if spec.int_inputs:
            assert np.array_equal(G, O), f"vp {spec.vp} integer sgemm must be exact"
            return
        A, B = inp["A"].astype(np.float64), inp["B"].astype(np.float64)
        scale = np.abs(spec.alpha) * (np.abs(A) @ np.abs(B))
        if spec.beta != 0:
            scale += np.abs(spec.beta * inp["C"].astype(np.float64))
        err = np.abs(G - O)
        assert (err <= sgemm_tol * scale + 1e-30).all(), (spec.vp, float((err / (scale + 1e-30)).max()))
        fro = np.linalg.norm(G - O) / (np.linalg.norm(O) + 1e-30)
        assert fro <= sgemm_tol, (spec.vp, "relative Frobenius error", fro)
    else:
        raise ValueError(k)


def inputs_for(specs, seed=W.BASE_SEED):
    return [W.make_inputs(s, seed) for s in specs]
