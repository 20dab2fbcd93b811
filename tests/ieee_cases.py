"""IEEE edge-value inputs for the fp32 "sgemm" implementations and their comparison with
the oracle (R9 "no FTZ/DAZ", R20 "special values").

The oracle (fp64 accumulation, one rounding, plain IEEE arithmetic in C) fixes what every
output must be: NaN where a NaN operand or an Inf*0 product or opposite infinities meet,
+-Inf where an infinite product dominates, and otherwise the finite value within the fp32
contract.  Inputs are built so that no FINITE fp32 partial sum overflows (one huge product
per output at most) -- fp32 accumulation overflowing where fp64 does not is outside every
fp32 GEMM's contract, FFMA's included.

Placement (A: M x K, B: K x N, the rest U[-1, 1)):
  row 0   A[0,3] = +Inf, with B[3,5] = 0                 -> C[0,5] NaN (Inf*0), C[0,j] +-Inf
  col 1   B[7,1] = -Inf                                   -> C[i,1] +-Inf (or NaN where row 0/5 meet it)
  row 2   A[2,10] = NaN (quiet, 0x7FC00000)               -> row NaN
  row 3   A[3,11] = NaN with payload only in the low 13 bits (0x7F800001) -> row NaN
  row 4   A[4,12] = NaN 0xFFFFFFFF (sign set, wraps an integer add)     -> row NaN
  row 5   A[5,13] = +Inf, B[13,6] = +Inf                 -> C[5,6] = +Inf*+Inf
  row 6   A[6,20] = FLT_MAX (0x7F7FFFFF: rounding to TF32 would overflow)   finite outputs
  row 7   A[7,21] = -3.4e38                                                finite outputs
  row 8   A[8,22] = 0x7F7FF000 (the rounding boundary to TF32 infinity)    finite outputs
  col 9   B[30,9] = FLT_MAX (B side), B[20..22, 9] = 0, A[6..8, 30] = 0     finite outputs
  row 10  A[10,:] subnormal (2^-140 scale)                -> tiny outputs
  col 10  B[:,10] subnormal (2^-140 scale)
  row 11  A[11,:] ~ 2^100, col 11 B[:,11] ~ 2^-131 (subnormal x large -> normal products)
  (12,12) A[12,:] = 0 except A[12,40] = 2^-130 (subnormal); B[40,12] = 2^120; B[k,12] = 0
          for k != 40 -> C[12,12] = 2^-10 exactly (a tensor core flushing subnormal inputs
          gives 0)
"""
from __future__ import annotations

import numpy as np

FLT_MAX = np.float32(np.finfo(np.float32).max)


def _bits(u: int) -> np.float32:
    return np.array([u], dtype=np.uint32).view(np.float32)[0]


def edge_inputs(M: int = 256, N: int = 256, K: int = 64, seed: int = 11, beta: float = 0.0):
    assert M >= 16 and N >= 16 and K >= 48
    g = np.random.default_rng(seed)
    A = (g.random((M, K), dtype=np.float32) * 2 - 1).astype(np.float32)
    B = (g.random((K, N), dtype=np.float32) * 2 - 1).astype(np.float32)
    A[0, 3] = np.inf
    B[3, 5] = 0.0
    B[7, 1] = -np.inf
    A[2, 10] = _bits(0x7FC00000)
    A[3, 11] = _bits(0x7F800001)
    A[4, 12] = _bits(0xFFFFFFFF)
    A[5, 13] = np.inf
    B[13, 6] = np.inf
    A[6, 20] = FLT_MAX
    A[7, 21] = np.float32(-3.4e38)
    A[8, 22] = _bits(0x7F7FF000)
    B[30, 9] = FLT_MAX
    B[20:23, 9] = 0.0
    A[6:9, 30] = 0.0
    sub = np.float32(2.0 ** -140)
    A[10, :] = (sub * (1 + g.random(K, dtype=np.float32)) * np.sign(g.random(K) - 0.5)).astype(np.float32)
    B[:, 10] = (sub * (1 + g.random(K, dtype=np.float32)) * np.sign(g.random(K) - 0.5)).astype(np.float32)
    A[11, :] = (np.float32(2.0 ** 100) * (1 + g.random(K, dtype=np.float32))).astype(np.float32)
    B[:, 11] = (np.float32(2.0 ** -131) * (1 + g.random(K, dtype=np.float32))).astype(np.float32)
    A[12, :] = 0.0
    A[12, 40] = np.float32(2.0 ** -130)
    B[:, 12] = 0.0
    B[40, 12] = np.float32(2.0 ** 120)
    out = {"A": A, "B": B}
    if beta != 0:
        out["C"] = (g.random((M, N), dtype=np.float32) * 2 - 1).astype(np.float32)
    return out


def tiny_mask(X: np.ndarray, lim: float = 2.0 ** -115) -> np.ndarray:
    """Nonzero finite operands below the tensor-core split's full-precision range."""
    a = np.abs(X.astype(np.float64))
    return np.isfinite(a) & (a > 0) & (a < lim)


def compare(G: np.ndarray, O: np.ndarray, A: np.ndarray, B: np.ndarray, alpha: float = 1.0, beta: float = 0.0,
            C_old=None, tol: float = 1e-5, tiny_coef: float = 0.0, inf_meets_zero_read: float = 0.0):
    """Classify every output against the oracle.

    Returns a dict: nan_mismatch / inf_mismatch / nonfinite_where_finite counts (with the
    first few positions) and, over the outputs the oracle gives finite, the max of
    |g - o| / bound with bound = tol * |alpha| (|A||B|)_ij + |beta C_ij| tol + (K + 1) 2^-149
    + tiny_coef * 2^-134 * sum_k (|a_ik| [b_kj tiny] + |b_kj| [a_ik tiny]).  ``tiny_coef`` = 0
    is the plain fp32 contract (R10 + the fp32 subnormal floor, R20); the tensor-core
    implementations state tiny_coef = 1 (R20).

    ``inf_meets_zero_read`` > 0: the one stated deviation of the tensor-core implementations
    (R20) -- an infinite operand times a nonzero operand below that magnitude (which the
    tensor core reads as 0: TF32's subnormal step is 2^-136) is Inf*0 = NaN there; where the
    oracle says +-Inf for such an output, NaN is accepted as well.
    """
    K = A.shape[1]
    G64, O64 = G.astype(np.float64), O.astype(np.float64)
    res = {}
    gn, on = np.isnan(G64), np.isnan(O64)
    exc = np.zeros(G.shape, dtype=bool)
    if inf_meets_zero_read:
        ia, ib = np.isinf(A).astype(np.float64), np.isinf(B).astype(np.float64)
        za, zb = (tiny_mask(A, inf_meets_zero_read).astype(np.float64),
                  tiny_mask(B, inf_meets_zero_read).astype(np.float64))
        exc = ((ia @ zb) + (za @ ib) > 0) & np.isinf(O64) & gn
    res["accepted_inf_as_nan"] = int(exc.sum())
    gn = gn & ~exc
    bad = np.argwhere(gn != on)
    res["nan_mismatch"] = int(len(bad))
    res["nan_mismatch_at"] = [tuple(map(int, x)) for x in bad[:6]]
    oi = np.isinf(O64) & ~exc
    bad = np.argwhere(oi & ~(G64 == O64))
    res["inf_mismatch"] = int(len(bad))
    res["inf_mismatch_at"] = [(tuple(map(int, x)), float(G64[tuple(x)]), float(O64[tuple(x)])) for x in bad[:6]]
    fin = np.isfinite(O64)
    bad = np.argwhere(fin & ~np.isfinite(G64))
    res["nonfinite_where_finite"] = int(len(bad))
    res["nonfinite_where_finite_at"] = [(tuple(map(int, x)), float(G64[tuple(x)])) for x in bad[:6]]
    A64 = np.where(np.isfinite(A), np.abs(A.astype(np.float64)), 0.0)
    B64 = np.where(np.isfinite(B), np.abs(B.astype(np.float64)), 0.0)
    bound = tol * abs(alpha) * (A64 @ B64) + (K + 1) * 2.0 ** -149
    if beta != 0 and C_old is not None:
        bound += tol * np.abs(beta * C_old.astype(np.float64))
    if tiny_coef:
        ta, tb = tiny_mask(A), tiny_mask(B)
        bound += tiny_coef * 2.0 ** -134 * abs(alpha) * (A64 @ tb.astype(np.float64) + ta.astype(np.float64) @ B64)
    ok = fin & np.isfinite(G64)
    ratio = np.where(ok, np.abs(G64 - O64) / bound, 0.0)
    res["max_err_over_bound"] = float(ratio.max()) if ok.any() else 0.0
    worst = np.unravel_index(int(np.argmax(ratio)), ratio.shape)
    res["worst_at"] = (tuple(map(int, worst)), float(G64[worst]), float(O64[worst]))
    res["over_bound"] = int((ratio > 1.0).sum())
    res["c_12_12"] = float(G64[12, 12]) if G.shape[0] > 12 and G.shape[1] > 12 else None
    return res


def passed(res) -> bool:
    return (res["nan_mismatch"] == 0 and res["inf_mismatch"] == 0 and res["nonfinite_where_finite"] == 0
            and res["over_bound"] == 0)


# What each fp32 "sgemm" implementation states (R20): NaN / +-Inf exactly as IEEE
# for all three (the tensor-core kernels recompute every output whose accumulator came out
# NaN in fp64 from the operands); finite outputs within the fp32 contract, the tensor-core
# splits adding the TF32/BF16 subnormal-granularity term for operands below 2^-115.
STATED = {"ffma": dict(tiny_coef=0.0),
          "3xtf32": dict(tiny_coef=1.0),
          "tf32bf16": dict(tiny_coef=1.0)}
