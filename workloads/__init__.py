"""Seeded synthetic inputs shared by the oracle tests, the GPU parity tests and bench.py.

This module is deliberately free of the method's arithmetic: it only draws random
numbers and lays out job specifications.  Neither the CUDA path (libsvp) nor the
oracle (oracle/) imports anything from here; the *callers* (tests, bench.py) draw
inputs here and hand the same arrays to both sides.

Recipe:
  * base seed 0x53565001; each (vp, stream) pair has its own PCG64 stream seeded
    by ``SeedSequence([seed, vp, stream])`` so inputs are identical whatever order
    or process draws them in (multi-rank runs draw only their own VPs).
  * vecadd a,b ~ U[-1,1) f32; saxpy x,y ~ U[-1,1), a_v ~ U[-2,2); hist256 bytes ~
    U{0..255} (or 90 % one value when skewed); Black-Scholes S~U[5,30],
    X~U[1,100], T~U[0.25,10], R=0.02, V=0.30 (CUDA-SDK ranges);
    SGEMM A,B ~ U[-1,1) (tolerance run) or integers U{-8..8} (exact run).
  * "1M", "4M", "64K-16M" are binary.  Ragged sizes are drawn
    log-uniform in [2^16, 2^24] as arbitrary integers, plus 8 adversarial sizes.
"""
from __future__ import annotations

import dataclasses
from typing import Dict, List, Optional

import numpy as np

BASE_SEED = 0x53565001

KERNELS = ("vecadd", "saxpy", "hist256", "blackscholes", "sgemm")
MEMBOUND = ("vecadd", "saxpy", "hist256", "blackscholes")

# stream ids (one PCG64 stream per (vp, purpose))
_S_SIZE, _S_A, _S_B, _S_C, _S_SCALAR = 1, 2, 3, 4, 5

ADVERSARIAL_SIZES = (2**16 + 1, 2**16 + 3, 4095, 4097, 2**24 - 1, 2**24, 1, 0)

BS_RISKFREE = 0.02
BS_VOLATILITY = 0.30


def rng(seed: int, vp: int, stream: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(np.random.SeedSequence([seed & 0xFFFFFFFF, vp, stream])))


def uniform_f32(g: np.random.Generator, n: int, lo: float, hi: float) -> np.ndarray:
    u = g.random(n, dtype=np.float32)
    return (np.float32(lo) + np.float32(hi - lo) * u).astype(np.float32, copy=False)


def int_f32(g: np.random.Generator, n: int, lo: int = -8, hi: int = 8) -> np.ndarray:
    return g.integers(lo, hi + 1, size=n, dtype=np.int32).astype(np.float32)


def dyadic_f32(g: np.random.Generator, n: int, bits: int = 10, kmax: int = 2**14) -> np.ndarray:
    """k / 2^bits with |k| < kmax: sums of two are exact in fp32 (pin for vecadd)."""
    k = g.integers(-kmax + 1, kmax, size=n, dtype=np.int32)
    return (k.astype(np.float32) / np.float32(2**bits)).astype(np.float32)


def bytes_u8(g: np.random.Generator, n: int, skew: bool = False) -> np.ndarray:
    d = g.integers(0, 256, size=n, dtype=np.uint8)
    if skew and n:
        hot = np.uint8(g.integers(0, 256))
        mask = g.random(n, dtype=np.float32) < np.float32(0.9)
        d[mask] = hot
    return d


def ragged_size(seed: int, vp: int, lo_log2: int = 16, hi_log2: int = 24) -> int:
    g = rng(seed, vp, _S_SIZE)
    return int(np.floor(2.0 ** g.uniform(lo_log2, hi_log2)))


@dataclasses.dataclass
class JobSpec:
    """One VP-kernel job: what a VP submits (kernel + size + scalar args)."""
    vp: int
    kernel: str
    n: int = 0                # elements (memory-bound kernels)
    M: int = 0                # SGEMM shape
    N: int = 0
    K: int = 0
    a: float = 0.0            # SAXPY scalar
    R: float = BS_RISKFREE    # Black-Scholes
    V: float = BS_VOLATILITY
    alpha: float = 1.0        # SGEMM
    beta: float = 0.0
    skew: bool = False        # hist256 skewed variant
    int_inputs: bool = False  # SGEMM exact (integer) run
    misalign: int = 0         # element offset of the buffer views (4-byte offset => non-16B-aligned)

    def input_bytes(self) -> int:
        if self.kernel in ("vecadd",):
            return 8 * self.n
        if self.kernel == "saxpy":
            return 8 * self.n
        if self.kernel == "hist256":
            return self.n
        if self.kernel == "blackscholes":
            return 12 * self.n
        if self.kernel in ("sgemm", "sgemm_tf32", "dgemm"):
            es = 8 if self.kernel == "dgemm" else 4
            return es * (self.M * self.K + self.K * self.N + (self.M * self.N if self.beta != 0 else 0))
        raise ValueError(self.kernel)

    def output_bytes(self) -> int:
        if self.kernel in ("vecadd", "saxpy"):
            return 4 * self.n
        if self.kernel == "hist256":
            return 1024
        if self.kernel == "blackscholes":
            return 8 * self.n
        if self.kernel in ("sgemm", "sgemm_tf32", "dgemm"):
            return (8 if self.kernel == "dgemm" else 4) * self.M * self.N
        raise ValueError(self.kernel)

    def algorithmic_bytes(self) -> int:
        """Bytes the kernel itself must move (SURVEY §8(d) roofline table)."""
        if self.kernel in ("vecadd", "saxpy"):
            return 12 * self.n
        if self.kernel == "hist256":
            return self.n + 1024
        if self.kernel == "blackscholes":
            return 20 * self.n
        if self.kernel in ("sgemm", "sgemm_tf32", "dgemm"):
            es = 8 if self.kernel == "dgemm" else 4
            return es * (self.M * self.K + self.K * self.N + self.M * self.N * (2 if self.beta != 0 else 1))
        raise ValueError(self.kernel)

    def flops(self) -> int:
        return 2 * self.M * self.N * self.K if self.kernel in ("sgemm", "sgemm_tf32", "dgemm") else 0


def _scalar_for(seed: int, spec: JobSpec) -> None:
    g = rng(seed, spec.vp, _S_SCALAR)
    if spec.kernel == "saxpy":
        spec.a = float(uniform_f32(g, 1, -2.0, 2.0)[0])


def make_inputs(spec: JobSpec, seed: int = BASE_SEED) -> Dict[str, np.ndarray]:
    """Host arrays for one job (inputs only; outputs are allocated by the caller)."""
    vp, n = spec.vp, spec.n
    k = spec.kernel
    if k == "vecadd":
        return {"a": uniform_f32(rng(seed, vp, _S_A), n, -1, 1),
                "b": uniform_f32(rng(seed, vp, _S_B), n, -1, 1)}
    if k == "saxpy":
        return {"x": uniform_f32(rng(seed, vp, _S_A), n, -1, 1),
                "y": uniform_f32(rng(seed, vp, _S_B), n, -1, 1)}
    if k == "hist256":
        return {"d": bytes_u8(rng(seed, vp, _S_A), n, spec.skew)}
    if k == "blackscholes":
        return {"S": uniform_f32(rng(seed, vp, _S_A), n, 5.0, 30.0),
                "X": uniform_f32(rng(seed, vp, _S_B), n, 1.0, 100.0),
                "T": uniform_f32(rng(seed, vp, _S_C), n, 0.25, 10.0)}
    if k == "dgemm":
        M, N, K = spec.M, spec.N, spec.K
        if spec.int_inputs:
            A = rng(seed, vp, _S_A).integers(-8, 9, M * K).astype(np.float64).reshape(M, K)
            B = rng(seed, vp, _S_B).integers(-8, 9, K * N).astype(np.float64).reshape(K, N)
        else:
            A = rng(seed, vp, _S_A).uniform(-1.0, 1.0, M * K).reshape(M, K)
            B = rng(seed, vp, _S_B).uniform(-1.0, 1.0, K * N).reshape(K, N)
        out = {"A": A, "B": B}
        if spec.beta != 0:
            out["C"] = rng(seed, vp, _S_C).uniform(-1.0, 1.0, M * N).reshape(M, N)
        return out
    if k in ("sgemm", "sgemm_tf32"):
        M, N, K = spec.M, spec.N, spec.K
        if spec.int_inputs:
            A = int_f32(rng(seed, vp, _S_A), M * K).reshape(M, K)
            B = int_f32(rng(seed, vp, _S_B), K * N).reshape(K, N)
        else:
            A = uniform_f32(rng(seed, vp, _S_A), M * K, -1, 1).reshape(M, K)
            B = uniform_f32(rng(seed, vp, _S_B), K * N, -1, 1).reshape(K, N)
        out = {"A": A, "B": B}
        if spec.beta != 0:  # C is an input only when beta != 0
            gen = int_f32 if spec.int_inputs else (lambda g, n: uniform_f32(g, n, -1, 1))
            out["C"] = gen(rng(seed, vp, _S_C), M * N).reshape(M, N)
        return out
    raise ValueError(k)


# --------------------------------------------------------------------------- configs
def make_inputs_many(specs, seed: int = BASE_SEED, threads: int = 0) -> List[Dict[str, np.ndarray]]:
    """make_inputs for many jobs on a thread pool (each job's streams are independent)."""
    from concurrent.futures import ThreadPoolExecutor
    import os
    threads = threads or min(32, len(os.sched_getaffinity(0)))
    with ThreadPoolExecutor(threads) as ex:
        return list(ex.map(lambda s: make_inputs(s, seed), specs))


def config_specs(cfg: int, seed: int = BASE_SEED, nvps: Optional[int] = None,
                 sgemm_int: bool = False, scale: int = 1) -> List[JobSpec]:
    """Job specs for BASELINE.json configs 1..5 (1-based, as listed there).

    ``scale`` divides every size (used to build reduced-size parity cases that keep
    the structure: ragged sizes, misaligned views, mixed kernels).
    """
    specs: List[JobSpec] = []
    if cfg == 1:
        for v in range(nvps or 2):
            specs.append(JobSpec(v, "vecadd", n=(1 << 20) // scale))
    elif cfg == 2:
        s = 512 // scale
        for v in range(nvps or 16):
            specs.append(JobSpec(v, "sgemm", M=s, N=s, K=s, int_inputs=sgemm_int))
    elif cfg == 3:
        for v in range(nvps or 64):
            k = MEMBOUND[v % 4]
            specs.append(JobSpec(v, k, n=(1 << 22) // scale))
    elif cfg in (4, 5):
        nv = nvps or (64 if cfg == 4 else 256)
        nk = 4 if cfg == 4 else 5
        kinds = MEMBOUND if cfg == 4 else KERNELS
        for v in range(nv):
            k = kinds[v % nk]
            if k == "sgemm":
                s = 2048 // scale
                specs.append(JobSpec(v, k, M=s, N=s, K=s, int_inputs=sgemm_int))
                continue
            if v < len(ADVERSARIAL_SIZES) and cfg == 4:
                n = ADVERSARIAL_SIZES[v]
            else:
                n = ragged_size(seed, v)
            n = n // scale if n > 16 else n
            specs.append(JobSpec(v, k, n=n, misalign=1 if (v % 8 == 7) else 0))
    else:
        raise ValueError(f"unknown config {cfg}")
    for s in specs:
        _scalar_for(seed, s)
        if s.kernel == "hist256":
            s.skew = (s.vp // 4) % 2 == 1 if cfg in (3, 4, 5) else False
    return specs


def table1_specs(nvps: int = 8, iters: int = 300, size: int = 320) -> List[JobSpec]:
    """The paper's Table 1 program on each of nvps VPs: `iters` multiplications of two
    size x size fp64 matrices, one job per multiplication in program
    order (vp-major list: VP v's jobs are consecutive)."""
    return [JobSpec(v, "dgemm", M=size, N=size, K=size) for v in range(nvps) for _ in range(iters)]


def mixed_small(nvps: int = 24, seed: int = BASE_SEED, max_n: int = 70000) -> List[JobSpec]:
    """A small mixed, ragged case (seconds for the oracle, several tiles + tails)."""
    specs = []
    for v in range(nvps):
        k = KERNELS[v % 5]
        if k == "sgemm":
            dims = [(128, 128, 128), (256, 128, 64), (96, 160, 72), (200, 136, 40)][v // 5 % 4]
            specs.append(JobSpec(v, k, M=dims[0], N=dims[1], K=dims[2]))
        else:
            g = rng(seed, v, _S_SIZE)
            n = int(g.integers(0, max_n)) if v % 7 else (v % 5)  # includes tiny / zero sizes
            specs.append(JobSpec(v, k, n=n, misalign=1 if v % 6 == 5 else 0))
        _scalar_for(seed, specs[-1])
    return specs
