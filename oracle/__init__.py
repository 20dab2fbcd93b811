"""oracle -- plain CPU reference for the SigmaVP hot path (TEST INFRASTRUCTURE ONLY).

Only ``tests/``, ``__graft_entry__.smoke()`` and bench.py's ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product path
(``paper_conf_dac_jungc15_b200``) never imports it and shares no code with it.

* ``svp_oracle.c`` -> ``liboracle.so``: per-VP guest kernels (vecadd, SAXPY,
  hist256, Black-Scholes, SGEMM) written as their plain definitions, each citing
  the passage it follows.
* :func:`run_jobs`: the paper's "emulation" baseline (Table 1):
  every VP runs its own jobs in program order, VPs spread over host threads
  (each VP single-threaded), no queue / matching / coalescing / streams.
* ``oracle.sched``: the timing models the paper states (Eq 7/8/9) and the
  brute-force schedules that pin the Re-scheduler and the Job Dispatcher.

Parity status per function is listed in DESIGN.md §"Oracle and pins"; the one
unpinned item is the per-VP attribution *inside* a coalesced launch (Profiler),
which is marked "parity unpinned" there and in ``oracle.sched``.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading
from concurrent.futures import ThreadPoolExecutor
from typing import Dict, List, Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "svp_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

_F32P = ctypes.POINTER(ctypes.c_float)
_F64P = ctypes.POINTER(ctypes.c_double)
_U8P = ctypes.POINTER(ctypes.c_uint8)
_U32P = ctypes.POINTER(ctypes.c_uint32)


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (no FMA contraction, no fast-math)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-std=c11",
                               "-shared", "-fPIC", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = ctypes.CDLL(_LIB)
            i64, i32, f32, f64 = ctypes.c_int64, ctypes.c_int32, ctypes.c_float, ctypes.c_double
            L.oracle_vecadd.argtypes = [i64, _F32P, _F32P, _F32P]
            L.oracle_saxpy.argtypes = [i64, f32, _F32P, _F32P]
            L.oracle_hist256.argtypes = [i64, _U8P, _U32P]
            L.oracle_blackscholes.argtypes = [i64, _F32P, _F32P, _F32P, f32, f32, _F32P, _F32P]
            L.oracle_blackscholes_f64.argtypes = [i64, _F64P, _F64P, _F64P, f64, f64, _F64P, _F64P]
            L.oracle_cnd_f32.argtypes = [f32]
            L.oracle_cnd_f32.restype = f32
            L.oracle_sgemm.argtypes = [i32, i32, i32, f32, _F32P, _F32P, f32, _F32P]
            L.oracle_sgemm_element.argtypes = [i32, i32, i32, f32, _F32P, _F32P, f32, f32, i32, i32]
            L.oracle_sgemm_element.restype = f32
            L.oracle_dgemm.argtypes = [i32, i32, i32, f64, _F64P, _F64P, f64, _F64P]
            L.oracle_dgemm.restype = None
            for f in ("oracle_vecadd", "oracle_saxpy", "oracle_hist256", "oracle_blackscholes",
                      "oracle_blackscholes_f64", "oracle_sgemm"):
                getattr(L, f).restype = None
            _lib = L
    return _lib


def _p(a: np.ndarray, t):
    assert a.flags["C_CONTIGUOUS"]
    return a.ctypes.data_as(t)


# ----------------------------------------------------------------- per-kernel wrappers
def vecadd(a: np.ndarray, b: np.ndarray) -> np.ndarray:
    c = np.empty_like(a)
    lib().oracle_vecadd(a.size, _p(a, _F32P), _p(b, _F32P), _p(c, _F32P))
    return c


def saxpy(a: float, x: np.ndarray, y: np.ndarray) -> np.ndarray:
    out = y.copy()
    lib().oracle_saxpy(x.size, ctypes.c_float(a), _p(x, _F32P), _p(out, _F32P))
    return out


def hist256(d: np.ndarray) -> np.ndarray:
    counts = np.empty(256, dtype=np.uint32)
    lib().oracle_hist256(d.size, _p(d, _U8P), _p(counts, _U32P))
    return counts


def blackscholes(S, X, T, R: float, V: float):
    call = np.empty_like(S)
    put = np.empty_like(S)
    lib().oracle_blackscholes(S.size, _p(S, _F32P), _p(X, _F32P), _p(T, _F32P),
                              ctypes.c_float(R), ctypes.c_float(V), _p(call, _F32P), _p(put, _F32P))
    return call, put


def blackscholes_f64(S, X, T, R: float, V: float):
    S, X, T = (np.ascontiguousarray(v, dtype=np.float64) for v in (S, X, T))
    call = np.empty_like(S)
    put = np.empty_like(S)
    lib().oracle_blackscholes_f64(S.size, _p(S, _F64P), _p(X, _F64P), _p(T, _F64P), R, V,
                                  _p(call, _F64P), _p(put, _F64P))
    return call, put


def cnd_f32(d: float) -> float:
    return float(lib().oracle_cnd_f32(ctypes.c_float(d)))


def sgemm(A: np.ndarray, B: np.ndarray, C: np.ndarray | None = None, alpha: float = 1.0,
          beta: float = 0.0) -> np.ndarray:
    M, K = A.shape
    K2, N = B.shape
    assert K == K2
    out = np.zeros((M, N), np.float32) if C is None else np.ascontiguousarray(C, dtype=np.float32).copy()
    lib().oracle_sgemm(M, N, K, ctypes.c_float(alpha), _p(A, _F32P), _p(B, _F32P),
                       ctypes.c_float(beta), _p(out, _F32P))
    return out


def sgemm_element(A, B, i: int, j: int, alpha: float = 1.0, beta: float = 0.0, c_old: float = 0.0) -> float:
    M, K = A.shape
    N = B.shape[1]
    return float(lib().oracle_sgemm_element(M, N, K, ctypes.c_float(alpha), _p(A, _F32P), _p(B, _F32P),
                                            ctypes.c_float(beta), ctypes.c_float(c_old), i, j))


def dgemm(A: np.ndarray, B: np.ndarray, C: np.ndarray | None = None, alpha: float = 1.0,
          beta: float = 0.0) -> np.ndarray:
    A = np.ascontiguousarray(A, dtype=np.float64)
    B = np.ascontiguousarray(B, dtype=np.float64)
    M, K = A.shape
    K2, N = B.shape
    assert K == K2
    out = np.zeros((M, N), np.float64) if C is None else np.ascontiguousarray(C, dtype=np.float64).copy()
    lib().oracle_dgemm(M, N, K, alpha, _p(A, _F64P), _p(B, _F64P), beta, _p(out, _F64P))
    return out


# ----------------------------------------------------------------- job-level runner
def run_job(spec, inputs: Dict[str, np.ndarray]) -> Dict[str, np.ndarray]:
    """One VP job, plain definition; returns the job's outputs by name."""
    k = spec.kernel
    if k == "vecadd":
        return {"c": vecadd(inputs["a"], inputs["b"])}
    if k == "saxpy":
        return {"y": saxpy(spec.a, inputs["x"], inputs["y"])}
    if k == "hist256":
        return {"counts": hist256(inputs["d"])}
    if k == "blackscholes":
        c, p = blackscholes(inputs["S"], inputs["X"], inputs["T"], spec.R, spec.V)
        return {"call": c, "put": p}
    if k == "dgemm":
        return {"C": dgemm(inputs["A"], inputs["B"], inputs.get("C") if spec.beta != 0 else None,
                           spec.alpha, spec.beta)}
    if k in ("sgemm", "sgemm_tf32"):  # same definition; the TF32 kernel has its own tolerance
        return {"C": sgemm(inputs["A"], inputs["B"], inputs.get("C") if spec.beta != 0 else None,
                           spec.alpha, spec.beta)}
    raise ValueError(k)


def run_jobs(specs: Sequence, inputs: Sequence[Dict[str, np.ndarray]], threads: int | None = None):
    """The emulation baseline: VPs run independently, each VP's jobs in program order.

    ``specs[i]`` / ``inputs[i]`` describe job i; jobs of one VP are executed in list
    order on one thread (a VP is single-threaded), distinct VPs in parallel.  Returns
    outputs aligned with ``specs``.  ctypes drops the GIL inside the C loops, so the
    host threads really run concurrently.
    """
    threads = threads or len(os.sched_getaffinity(0))
    by_vp: Dict[int, List[int]] = {}
    for i, s in enumerate(specs):
        by_vp.setdefault(s.vp, []).append(i)
    results: List[Dict[str, np.ndarray]] = [None] * len(specs)  # type: ignore

    def one_vp(idx: List[int]):
        for i in idx:
            results[i] = run_job(specs[i], inputs[i])

    with ThreadPoolExecutor(max_workers=threads) as ex:
        list(ex.map(one_vp, by_vp.values()))
    return results
