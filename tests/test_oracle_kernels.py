"""Pins for the oracle's guest kernels (CPU only).

Each test pins an oracle function to something other than itself: exact closed
forms, textbook tables, library routines on special cases, or brute force on tiny
inputs -- chosen so a dropped term / wrong sign / transposed operand fails.
"""
from fractions import Fraction

import numpy as np
import pytest

import oracle
import workloads as W


# ------------------------------------------------------------------ vecadd
def test_vecadd_dyadic_exact():
    g = W.rng(1, 0, 2)
    a = W.dyadic_f32(g, 10007)
    b = W.dyadic_f32(g, 10007)
    exact = (a.astype(np.float64) + b.astype(np.float64))  # exact: |k| < 2^15 over 2^10
    assert np.array_equal(oracle.vecadd(a, b).astype(np.float64), exact)


def test_vecadd_matches_ieee_add():
    g = W.rng(2, 0, 2)
    a = W.uniform_f32(g, 4099, -1, 1)
    b = W.uniform_f32(g, 4099, -1e-3, 1e3)
    assert np.array_equal(oracle.vecadd(a, b), np.add(a, b, dtype=np.float32))


def test_vecadd_empty_and_order():
    a = np.array([1.0, 2.0, 3.0], np.float32)
    b = np.array([10.0, 20.0, 30.0], np.float32)
    assert oracle.vecadd(a, b).tolist() == [11.0, 22.0, 33.0]
    assert oracle.vecadd(np.zeros(0, np.float32), np.zeros(0, np.float32)).size == 0


# ------------------------------------------------------------------ SAXPY
def test_saxpy_integer_exact():
    g = W.rng(3, 0, 2)
    x = g.integers(-1024, 1025, 5000).astype(np.float32)
    y = g.integers(-1024, 1025, 5000).astype(np.float32)
    out = oracle.saxpy(-7.0, x, y)
    assert np.array_equal(out.astype(np.int64), (-7 * x.astype(np.int64) + y.astype(np.int64)))


def _round_f32(fr: Fraction) -> np.float32:
    # correctly rounded (nearest-even) fraction -> float32
    f = np.float32(float(fr))  # float(fr) is correctly rounded to f64; fix double rounding below
    cands = [np.nextafter(f, np.float32(-np.inf)), f, np.nextafter(f, np.float32(np.inf))]
    best = min(cands, key=lambda c: (abs(Fraction(float(c)) - fr), int(np.frombuffer(c.tobytes(), np.uint32)[0]) & 1))
    return best


def test_saxpy_single_rounding_vs_exact_fraction():
    """fma semantics: one rounding of the exact a*x+y (a separate mul+add would differ)."""
    g = W.rng(4, 0, 2)
    x = W.uniform_f32(g, 400, -1, 1)
    y = W.uniform_f32(g, 400, -1, 1)
    a = np.float32(1.2345678)
    out = oracle.saxpy(float(a), x, y)
    for i in range(400):
        exact = Fraction(float(a)) * Fraction(float(x[i])) + Fraction(float(y[i]))
        assert out[i] == _round_f32(exact), i
    # at least one element where unfused mul-then-add differs (proves the fma is there)
    unfused = (a * x).astype(np.float32) + y
    assert np.any(unfused != out)


# ------------------------------------------------------------------ hist256
def test_hist_invariants_and_patterns():
    m = 37
    d = (np.arange(256 * m) % 256).astype(np.uint8)
    c = oracle.hist256(d)
    assert np.all(c == m)
    z = np.zeros(1001, np.uint8)
    cz = oracle.hist256(z)
    assert cz[0] == 1001 and cz[1:].sum() == 0
    assert oracle.hist256(np.zeros(0, np.uint8)).sum() == 0


@pytest.mark.parametrize("skew", [False, True])
def test_hist_vs_bincount(skew):
    d = W.bytes_u8(W.rng(5, 1, 2), 123457, skew)
    c = oracle.hist256(d)
    assert c.sum() == d.size
    assert np.array_equal(c, np.bincount(d, minlength=256).astype(np.uint32))


def test_hist_brute_force_tiny():
    from collections import Counter
    d = np.array([3, 255, 3, 0, 7, 7, 7], np.uint8)
    c = oracle.hist256(d)
    cnt = Counter(d.tolist())
    assert all(c[b] == cnt.get(b, 0) for b in range(256))


# ------------------------------------------------------------------ Black-Scholes
def test_cnd_against_table(golden):
    for x, nx in golden("normal_cdf_table.txt"):
        assert abs(oracle.cnd_f32(float(x)) - float(nx)) < 2e-7, x  # A&S 7.5e-8 + fp32 rounding


def test_cnd_symmetry():
    for x in np.linspace(-6, 6, 241):
        s = oracle.cnd_f32(float(x)) + oracle.cnd_f32(float(-x))
        assert abs(s - 1.0) < 2e-7


def test_blackscholes_textbook(golden):
    for S, X, T, R, V, call, put, tol, _src in golden("blackscholes_textbook.txt"):
        S, X, T, R, V, call, put, tol = map(float, (S, X, T, R, V, call, put, tol))
        c64, p64 = oracle.blackscholes_f64(np.array([S]), np.array([X]), np.array([T]), R, V)
        assert abs(c64[0] - call) <= tol and abs(p64[0] - put) <= tol
        c32, p32 = oracle.blackscholes(*(np.array([v], np.float32) for v in (S, X, T)), R, V)
        assert abs(c32[0] - call) <= max(tol, 1e-5 * S)
        assert abs(p32[0] - put) <= max(tol, 1e-5 * S)


def test_blackscholes_put_call_parity_and_f64():
    spec = W.JobSpec(0, "blackscholes", n=20000)
    inp = W.make_inputs(spec, seed=11)
    call, put = oracle.blackscholes(inp["S"], inp["X"], inp["T"], spec.R, spec.V)
    S, X, T = (inp[k].astype(np.float64) for k in "SXT")
    disc = X * np.exp(-spec.R * T)
    scale = np.maximum(S, disc)
    # C - P = S - X e^{-RT} for any CND with N(-d) = 1 - N(d)
    assert np.max(np.abs((call - put) - (S - disc)) / scale) < 1e-5
    c64, p64 = oracle.blackscholes_f64(S, X, T, float(np.float32(spec.R)), float(np.float32(spec.V)))
    assert np.max(np.abs(call - c64) / scale) < 1e-5
    assert np.max(np.abs(put - p64) / scale) < 1e-5
    # prices obey no-arbitrage bounds
    assert np.all(call >= -1e-4 * scale) and np.all(put >= -1e-4 * scale)
    assert np.all(call <= S + 1e-4 * scale)


# ------------------------------------------------------------------ SGEMM
def test_sgemm_integer_exact_vs_int_matmul():
    spec = W.JobSpec(0, "sgemm", M=67, N=45, K=129, int_inputs=True)
    inp = W.make_inputs(spec, seed=5)
    C = oracle.sgemm(inp["A"], inp["B"])
    ref = inp["A"].astype(np.int64) @ inp["B"].astype(np.int64)
    assert np.array_equal(C.astype(np.int64), ref)


def test_sgemm_identity_and_transposition():
    g = W.rng(6, 0, 2)
    A = W.uniform_f32(g, 24 * 16, -1, 1).reshape(24, 16)
    assert np.array_equal(oracle.sgemm(A, np.eye(16, dtype=np.float32)), A)
    # non-square + asymmetric: A (2x3) B (3x2) by hand
    A = np.array([[1, 2, 3], [4, 5, 6]], np.float32)
    B = np.array([[7, 8], [9, 10], [11, 12]], np.float32)
    assert oracle.sgemm(A, B).tolist() == [[58, 64], [139, 154]]


def test_sgemm_alpha_beta():
    A = np.array([[1, 2], [3, 4]], np.float32)
    B = np.array([[5, 6], [7, 8]], np.float32)
    C = np.array([[1, -1], [2, 0.5]], np.float32)
    out = oracle.sgemm(A, B, C, alpha=2.0, beta=-3.0)
    assert out.tolist() == [[2 * 19 - 3, 2 * 22 + 3], [2 * 43 - 6, 2 * 50 - 1.5]]


def test_sgemm_random_near_exact():
    g = W.rng(7, 0, 2)
    M, N, K = 33, 70, 300
    A = W.uniform_f32(g, M * K, -1, 1).reshape(M, K)
    B = W.uniform_f32(g, K * N, -1, 1).reshape(K, N)
    C = oracle.sgemm(A, B)
    ref = A.astype(np.float64) @ B.astype(np.float64)
    # fp64 accumulation then one rounding: within 1 ulp of fp32 of the exact value
    assert np.all(np.abs(C - ref) <= np.spacing(np.abs(ref).astype(np.float32)) * 1.0 + 1e-12)
    for (i, j) in [(0, 0), (M - 1, N - 1), (5, 17)]:
        assert oracle.sgemm_element(A, B, i, j) == C[i, j]


def test_sgemm_element_alpha_beta_against_int64_closed_form():
    """oracle_sgemm_element's beta / c_old branch (the checker of every full-size sampled
    GEMM output) against the int64 closed form alpha * sum_k a_ik b_kj + beta * c_old, with
    integer operands small enough that every value is exact in fp32 -- a dropped beta term,
    a sign slip or a transposed index fails it.  beta == 0 must not read c_old (BLAS: C is
    not an input then), so a NaN c_old is ignored."""
    g = np.random.default_rng(17)
    M, N, K = 37, 53, 61
    A = g.integers(-8, 9, (M, K)).astype(np.float32)
    B = g.integers(-8, 9, (K, N)).astype(np.float32)
    Cold = g.integers(-100, 101, (M, N)).astype(np.float32)
    exact = A.astype(np.int64) @ B.astype(np.int64)
    for alpha, beta in [(1.0, 0.0), (2.0, -3.0), (-1.0, 0.5), (0.0, 1.0), (3.0, 2.0)]:
        for (i, j) in [(0, 0), (M - 1, N - 1), (5, 17), (36, 0), (0, 52)]:
            want = alpha * float(exact[i, j]) + (beta * float(Cold[i, j]) if beta else 0.0)
            got = oracle.sgemm_element(A, B, i, j, alpha, beta, float(Cold[i, j]))
            assert got == want, (alpha, beta, i, j, got, want)
            assert oracle.sgemm_element(A, B, i, j, alpha, beta, float(Cold[i, j])) == \
                oracle.sgemm(A, B, Cold, alpha, beta)[i, j]
    assert oracle.sgemm_element(A, B, 3, 4, 1.0, 0.0, float("nan")) == float(exact[3, 4])


def test_sgemm_ieee_special_values():
    """The oracle's own IEEE behaviour (R20): Inf*0 = NaN, Inf*x = +-Inf, Inf*Inf = Inf,
    Inf + -Inf = NaN, a NaN operand poisons its row, subnormal operands are exact (fp64)."""
    A = np.array([[np.inf, 1.0], [np.inf, -1.0], [np.nan, 0.0], [2.0 ** -140, 0.0]], np.float32)
    B = np.array([[0.0, 2.0, np.inf], [1.0, 1.0, np.inf]], np.float32)
    C = oracle.sgemm(A, B)
    assert np.isnan(C[0, 0])                      # Inf*0 + 1*1
    assert C[0, 1] == np.inf                      # Inf*2 + 1
    assert C[0, 2] == np.inf                      # Inf*Inf + Inf
    assert np.isnan(C[1, 2])                      # Inf*Inf + (-1)*Inf
    assert np.isnan(C[2]).all()                   # NaN row
    assert C[3, 1] == np.float32(2.0 ** -139)     # subnormal * 2, exact


# ------------------------------------------------------------------ job runner
def test_run_jobs_independent_per_vp():
    specs = W.mixed_small(nvps=10, max_n=5000)
    inputs = [W.make_inputs(s) for s in specs]
    res = oracle.run_jobs(specs, inputs, threads=4)
    for s, inp, r in zip(specs, inputs, res):
        single = oracle.run_job(s, inp)
        for k in single:
            assert np.array_equal(single[k], r[k])


# ------------------------------------------------------------------ DGEMM (Table 1 guest)
def test_dgemm_integer_exact_and_hand_case():
    spec = W.JobSpec(0, "dgemm", M=37, N=29, K=65, int_inputs=True)
    inp = W.make_inputs(spec, seed=9)
    C = oracle.dgemm(inp["A"], inp["B"])
    assert np.array_equal(C.astype(np.int64), inp["A"].astype(np.int64) @ inp["B"].astype(np.int64))
    A = np.array([[1, 2, 3], [4, 5, 6]], np.float64)
    B = np.array([[7, 8], [9, 10], [11, 12]], np.float64)
    assert oracle.dgemm(A, B).tolist() == [[58, 64], [139, 154]]
    Cin = np.array([[1, -1], [2, 0.5]])
    assert oracle.dgemm(A, B, Cin, 2.0, -3.0).tolist() == [[113, 131], [272, 306.5]]


def test_dgemm_identity_and_near_exact():
    g = W.rng(8, 0, 2)
    A = g.uniform(-1, 1, (40, 33))
    assert np.array_equal(oracle.dgemm(A, np.eye(33)), A)
    B = g.uniform(-1, 1, (33, 50))
    # extended-precision accumulation: within 1 ulp of the correctly rounded product
    from fractions import Fraction
    C = oracle.dgemm(A, B)
    for (i, j) in [(0, 0), (39, 49), (7, 21)]:
        exact = sum(Fraction(float(A[i, k])) * Fraction(float(B[k, j])) for k in range(33))
        assert abs(Fraction(float(C[i, j])) - exact) <= Fraction(np.spacing(abs(float(exact)))), (i, j)


# ------------------------------------------------------------------ property tests
from hypothesis import given, settings  # noqa: E402
from hypothesis import strategies as st  # noqa: E402


@settings(max_examples=60, deadline=None)
@given(M=st.integers(0, 9), N=st.integers(0, 9), K=st.integers(0, 9), seed=st.integers(0, 2**31 - 1),
       alpha=st.sampled_from([1.0, -2.0, 0.5]), beta=st.sampled_from([0.0, 1.0, -0.25]))
def test_sgemm_random_tiny_shapes_exact(M, N, K, seed, alpha, beta):
    """Random tiny shapes (incl. empty), integer operands in [-8, 8]: the oracle's SGEMM equals
    alpha * (int64 matmul) + beta * C exactly (every intermediate is a small dyadic)."""
    g = np.random.default_rng(seed)
    A = g.integers(-8, 9, size=(M, K)).astype(np.float32)
    B = g.integers(-8, 9, size=(K, N)).astype(np.float32)
    C = g.integers(-8, 9, size=(M, N)).astype(np.float32)
    want = alpha * (A.astype(np.int64) @ B.astype(np.int64)).astype(np.float64) + beta * C.astype(np.float64)
    got = oracle.sgemm(A, B, C.copy(), alpha, beta)
    assert got.shape == (M, N)
    assert np.array_equal(got.astype(np.float64), want)


@settings(max_examples=60, deadline=None)
@given(data=st.binary(min_size=0, max_size=600))
def test_hist_random_bytes_brute_force(data):
    """Arbitrary byte strings (incl. empty): counts equal a pure-Python tally and sum to n."""
    d = np.frombuffer(data, dtype=np.uint8)
    want = [0] * 256
    for x in data:
        want[x] += 1
    got = oracle.hist256(d)
    assert list(got) == want and int(got.sum()) == len(data)


@settings(max_examples=60, deadline=None)
@given(n=st.integers(0, 300), seed=st.integers(0, 2**31 - 1), a=st.integers(-64, 64))
def test_saxpy_random_integer_exact(n, seed, a):
    """Integer-valued a, x, y (|.| <= 2^10): y' = a x + y is exact in fp32, so the oracle must
    match the exact integer result for any length (incl. 0)."""
    g = np.random.default_rng(seed)
    x = g.integers(-1024, 1025, size=n).astype(np.float32)
    y = g.integers(-1024, 1025, size=n).astype(np.float32)
    want = a * x.astype(np.int64) + y.astype(np.int64)
    assert np.array_equal(oracle.saxpy(float(a), x, y.copy()).astype(np.int64), want)
