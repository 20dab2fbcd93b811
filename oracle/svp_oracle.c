/*
 * svp_oracle.c -- plain, slow, obviously-correct CPU reference for the SigmaVP hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  It shares no code,
 * header, table or constant generator with the CUDA path (paper_conf_dac_jungc15_b200/csrc),
 * and neither side includes or links the other.
 *
 * What it computes: Kernel Coalescing and Kernel Interleaving are
 * execution transformations that must leave every VP's result unchanged -- after a
 * coalesced run "the resulting data are properly divided to be copied from the GPU
 * device back to the host memory addresses" (§3 "Coalescing
 * Identical Kernels").  The oracle is therefore the plain per-VP definition of each
 * guest kernel, mirroring the paper's "CUDA Emul. on CPU" baseline (Table 1,
 * PAPER.md L737-747): each VP's job runs alone, in program order, with plain loops.
 *
 * Precision: the paper fixes none for these kernels except Table 1's fp64 matmul
 * (PAPER.md L818-820).  BASELINE.json fixes fp32 guest data, so the guest kernels are
 * fp32 with the single-rounding semantics spelled out per function; SGEMM
 * accumulates in fp64 (exact float*float products) and rounds once, and an fp64
 * Black-Scholes twin with the exact normal CDF backs the oracle's own pins.
 *
 * Build: gcc -O2 -ffp-contract=off -fno-fast-math -shared -fPIC (no FMA contraction,
 * no reassociation; fmaf() is called explicitly where the definition has one).
 */
#include <math.h>
#include <stddef.h>
#include <stdint.h>
#include <string.h>
#include <stdlib.h>

/* vectorAdd (CUDA SDK; Fig 10): c[i] = a[i] + b[i], one fp32
 * rounding per element. */
void oracle_vecadd(int64_t n, const float* a, const float* b, float* c) {
    for (int64_t i = 0; i < n; ++i) c[i] = a[i] + b[i];
}

/* SAXPY (BASELINE.json guest kernel): y[i] = fma(a, x[i], y[i]) with a
 * single rounding (IEEE-754 fusedMultiplyAdd, C99 fmaf). */
void oracle_saxpy(int64_t n, float a, const float* x, float* y) {
    for (int64_t i = 0; i < n; ++i) y[i] = fmaf(a, x[i], y[i]);
}

/* 256-bin histogram (BASELINE.json): counts[b] = #{i : d[i] == b},
 * b in [0,256).  The result overwrites counts. */
void oracle_hist256(int64_t n, const uint8_t* d, uint32_t* counts) {
    for (int b = 0; b < 256; ++b) counts[b] = 0;
    for (int64_t i = 0; i < n; ++i) counts[d[i]] += 1u;
}

/* Cumulative normal distribution, polynomial approximation of Abramowitz & Stegun
 * 26.2.17 as used by the CUDA SDK BlackScholes sample (the paper
 * names the SDK BlackScholes program):
 *   K = 1/(1 + 0.2316419 |d|)
 *   cnd = RSQRT2PI * exp(-d^2/2) * K*(A1 + K*(A2 + K*(A3 + K*(A4 + K*A5))))
 *   if d > 0: cnd = 1 - cnd                                                        */
static float cnd_as_f32(float d) {
    const float A1 = 0.31938153f, A2 = -0.356563782f, A3 = 1.781477937f,
                A4 = -1.821255978f, A5 = 1.330274429f;
    const float RSQRT2PI = 0.39894228040143267793994605993438f;
    float K = 1.0f / (1.0f + 0.2316419f * fabsf(d));
    float cnd = RSQRT2PI * expf(-0.5f * d * d) *
                (K * (A1 + K * (A2 + K * (A3 + K * (A4 + K * A5)))));
    if (d > 0) cnd = 1.0f - cnd;
    return cnd;
}

/* Black-Scholes European call/put:
 *   d1 = (ln(S/X) + (R + V^2/2) T) / (V sqrt(T)),  d2 = d1 - V sqrt(T)
 *   Call = S N(d1) - X e^{-RT} N(d2),   Put = X e^{-RT} (1 - N(d2)) - S (1 - N(d1))
 * fp32 throughout, libm expf/logf/sqrtf, N = A&S CND above. */
void oracle_blackscholes(int64_t n, const float* S, const float* X, const float* T,
                         float R, float V, float* call, float* put) {
    for (int64_t i = 0; i < n; ++i) {
        float s = S[i], x = X[i], t = T[i];
        float sqrtT = sqrtf(t);
        float d1 = (logf(s / x) + (R + 0.5f * V * V) * t) / (V * sqrtT);
        float d2 = d1 - V * sqrtT;
        float N1 = cnd_as_f32(d1), N2 = cnd_as_f32(d2);
        float expRT = expf(-R * t);
        call[i] = s * N1 - x * expRT * N2;
        put[i] = x * expRT * (1.0f - N2) - s * (1.0f - N1);
    }
}

/* fp64 twin with the exact normal CDF N(x) = erfc(-x/sqrt 2)/2 -- used only to pin the
 * oracle itself against textbook values (never compared with the GPU). */
void oracle_blackscholes_f64(int64_t n, const double* S, const double* X, const double* T,
                             double R, double V, double* call, double* put) {
    for (int64_t i = 0; i < n; ++i) {
        double s = S[i], x = X[i], t = T[i];
        double d1 = (log(s / x) + (R + 0.5 * V * V) * t) / (V * sqrt(t));
        double d2 = d1 - V * sqrt(t);
        double N1 = 0.5 * erfc(-d1 / sqrt(2.0)), N2 = 0.5 * erfc(-d2 / sqrt(2.0));
        call[i] = s * N1 - x * exp(-R * t) * N2;
        put[i] = x * exp(-R * t) * (1.0 - N2) - s * (1.0 - N1);
    }
}

/* The A&S CND alone (so tests can pin it against tabulated N(x)). */
float oracle_cnd_f32(float d) { return cnd_as_f32(d); }

/* SGEMM (the paper's matmul guest, Table 1, at BASELINE.json's fp32):
 *   C = alpha * A B + beta * C,  A: MxK, B: KxN, C: MxN, all row-major, dense.
 * The "naive triple loop" of BASELINE.json: for each (i, j), sum_k A[i,k] B[k,j] in
 * ascending k with an fp64 accumulator (float*float is exact in fp64), then
 * alpha*acc + beta*C[i,j] in fp64 and a single rounding to fp32.  The loop is written
 * i-k-j so it streams rows; the per-element summation order is the same as i-j-k. */
void oracle_sgemm(int32_t M, int32_t N, int32_t K, float alpha, const float* A,
                  const float* B, float beta, float* C) {
    double* acc = (double*)malloc(sizeof(double) * (size_t)(N > 0 ? N : 1));
    for (int32_t i = 0; i < M; ++i) {
        for (int32_t j = 0; j < N; ++j) acc[j] = 0.0;
        for (int32_t k = 0; k < K; ++k) {
            double a = (double)A[(size_t)i * K + k];
            const float* brow = B + (size_t)k * N;
            for (int32_t j = 0; j < N; ++j) acc[j] += a * (double)brow[j];
        }
        float* crow = C + (size_t)i * N;
        for (int32_t j = 0; j < N; ++j) {
            double r = (double)alpha * acc[j];
            if (beta != 0.0f) r += (double)beta * (double)crow[j];
            crow[j] = (float)r;
        }
    }
    free(acc);
}

/* One output element of the SGEMM definition above -- lets parity tests at full size
 * check sampled outputs one by one without running the whole product. */
float oracle_sgemm_element(int32_t M, int32_t N, int32_t K, float alpha, const float* A,
                           const float* B, float beta, float c_old, int32_t i, int32_t j) {
    (void)M;
    double acc = 0.0;
    for (int32_t k = 0; k < K; ++k) acc += (double)A[(size_t)i * K + k] * (double)B[(size_t)k * N + j];
    double r = (double)alpha * acc;
    if (beta != 0.0f) r += (double)beta * (double)c_old;
    return (float)r;
}

/* DGEMM -- the paper's own matmul guest at its stated precision (Table 1: "multiplies
 * 300 times two 320 x 320 matrices of double-precision numbers"):
 *   C = alpha * A B + beta * C, fp64, row-major.  Plain i-k-j loop with an extended-
 * precision (x87 long double, 64-bit mantissa) accumulator per output element, ascending
 * k, then alpha*acc + beta*C in long double and one rounding to double. */
void oracle_dgemm(int32_t M, int32_t N, int32_t K, double alpha, const double* A, const double* B,
                  double beta, double* C) {
    long double* acc = (long double*)malloc(sizeof(long double) * (size_t)(N > 0 ? N : 1));
    for (int32_t i = 0; i < M; ++i) {
        for (int32_t j = 0; j < N; ++j) acc[j] = 0.0L;
        for (int32_t k = 0; k < K; ++k) {
            long double a = (long double)A[(size_t)i * K + k];
            const double* brow = B + (size_t)k * N;
            for (int32_t j = 0; j < N; ++j) acc[j] += a * (long double)brow[j];
        }
        double* crow = C + (size_t)i * N;
        for (int32_t j = 0; j < N; ++j) {
            long double r = (long double)alpha * acc[j];
            if (beta != 0.0) r += (long double)beta * (long double)crow[j];
            crow[j] = (double)r;
        }
    }
    free(acc);
}
