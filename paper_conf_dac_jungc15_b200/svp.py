"""Thin ctypes binding of libsvp (include/svp.h) -- argument marshalling only.

Every step of the hot path (Kernel Match, Dispatcher, Re-scheduler, coalesced
sm_100a kernels, interleaved copies, Profiler) runs inside libsvp.so; this module only
converts Python values to the C structs.  There is no fallback: if libsvp.so is
missing or fails to load, :func:`load` raises.
"""
from __future__ import annotations

import ctypes as C
import os
import struct
import threading
from typing import Dict, Iterable, List, Optional, Sequence, Tuple

_PKG = os.path.dirname(os.path.abspath(__file__))
# SVP_LIB: load another build of the same library (the host-sanitizer builds of
# scripts/host_sanitizers.sh); it is then used as is, never rebuilt.
LIB_PATH = os.environ.get("SVP_LIB") or os.path.join(_PKG, "libsvp.so")

SVP_OK, SVP_E_INVAL, SVP_E_NOMEM, SVP_E_CUDA, SVP_E_NOKERNEL, SVP_E_STATE, SVP_E_TIMEOUT, SVP_E_UNSUPPORTED = (
    0, -1, -2, -3, -4, -5, -6, -7)
STATUS_NAMES = {0: "SVP_OK", -1: "SVP_E_INVAL", -2: "SVP_E_NOMEM", -3: "SVP_E_CUDA", -4: "SVP_E_NOKERNEL",
                -5: "SVP_E_STATE", -6: "SVP_E_TIMEOUT", -7: "SVP_E_UNSUPPORTED"}
DIR_IN, DIR_OUT, DIR_INOUT = 1, 2, 3
MEM_DEVICE, MEM_HOST_PINNED = 0, 1
OP_H2D, OP_KERNEL, OP_D2H = 0, 1, 2
SGEMM_FFMA, SGEMM_3XTF32, SGEMM_TF32BF16 = 0, 1, 2
KERNEL_EW_MIX = 8  # heterogeneous elementwise launch (cfg hetero): plan/kernel-stats id only
TABLE_GLOBAL, TABLE_PARAM = 0, 1
MAX_BUFS, MAX_ARGS = 5, 64

# ABI symbols declared in include/svp.h (tests check every one is exported)
EXPORTS = ("svp_config_default", "svp_init", "svp_finalize", "svp_last_error", "svp_abi_version",
           "svp_register_kernel", "svp_submit", "svp_submit_batch", "svp_flush", "svp_vp_device",
           "svp_assign_vps", "svp_lpt_partition", "svp_profile", "svp_reset_profile", "svp_kernel_stats_get",
           "svp_flush_stats_get", "svp_plan_size", "svp_plan_get", "svp_wait", "svp_start_dispatcher",
           "svp_stop_dispatcher", "svp_ipc_serve", "svp_ipc_server_stats", "svp_ipc_shutdown", "svp_ipc_connect",
           "svp_ipc_disconnect", "svp_ipc_alloc", "svp_ipc_submit", "svp_ipc_wait", "svp_kernel_lookup",
           "svp_plan_op_detail", "svp_device_stats_get", "svp_host_alloc", "svp_host_free",
           "svp_flush_async", "svp_flush_wait")


class svp_config(C.Structure):
    _fields_ = [("num_gpus", C.c_int32), ("device_ids", C.POINTER(C.c_int32)), ("streams_per_gpu", C.c_int32),
                ("coalesce", C.c_int32), ("interleave", C.c_int32), ("max_chunks", C.c_int32),
                ("arena_bytes", C.c_uint64), ("profile_level", C.c_int32), ("sync_each_job", C.c_int32),
                ("dry_run", C.c_int32), ("flush_timeout_ms", C.c_int32), ("validate_ptrs", C.c_int32),
                ("sgemm_impl", C.c_int32),
                ("external_streams", C.POINTER(C.c_void_p)), ("hbm_gbps", C.c_double), ("pcie_gbps", C.c_double),
                ("ffma_tflops", C.c_double), ("launch_us", C.c_double), ("hetero", C.c_int32),
                ("graph", C.c_int32), ("table_mode", C.c_int32), ("sgemm_kchunk", C.c_int32)]


class svp_buf(C.Structure):
    _fields_ = [("ptr", C.c_void_p), ("bytes", C.c_uint64), ("dir", C.c_int32), ("mem", C.c_int32)]


class svp_job_desc(C.Structure):
    _fields_ = [("vp", C.c_int32), ("kernel", C.c_int32), ("args_bytes", C.c_uint32), ("nbufs", C.c_int32),
                ("args", C.c_uint8 * MAX_ARGS), ("bufs", svp_buf * MAX_BUFS)]


class svp_ipc_buf(C.Structure):
    _fields_ = [("offset", C.c_uint64), ("bytes", C.c_uint64), ("dir", C.c_int32), ("_pad", C.c_int32)]


class svp_vp_profile(C.Structure):
    _fields_ = [("jobs", C.c_uint64), ("kernel_ns", C.c_double), ("h2d_ns", C.c_double), ("d2h_ns", C.c_double),
                ("bytes_kernel", C.c_uint64), ("bytes_h2d", C.c_uint64), ("bytes_d2h", C.c_uint64),
                ("flops", C.c_double), ("launches", C.c_uint64)]


class svp_kernel_stats(C.Structure):
    _fields_ = [("launches", C.c_uint64), ("total_ns", C.c_double), ("bytes", C.c_double), ("flops", C.c_double),
                ("max_ns", C.c_double)]


class svp_flush_stats(C.Structure):
    _fields_ = [(n, C.c_uint64) for n in ("jobs", "groups", "chunks", "launches", "levels", "h2d_bytes",
                                          "d2h_bytes", "table_bytes", "table_uploads")] + \
               [(n, C.c_double) for n in ("host_plan_ns", "host_issue_ns", "host_total_ns", "device_ns",
                                          "sim_makespan_ns", "sim_serial_ns")] + \
               [(n, C.c_uint64) for n in ("plan_reused", "graph_replays", "kernel_launches")]


class svp_device_stats(C.Structure):
    _fields_ = [("ordinal", C.c_int32), ("vps", C.c_int32), ("est_load_ns", C.c_double), ("flushes", C.c_uint64),
                ("jobs", C.c_uint64), ("device_ns", C.c_double), ("kernel_ns", C.c_double),
                ("last_device_ns", C.c_double), ("numa_node", C.c_int32), ("worker_cpu_pinned", C.c_int32)]


class svp_plan_op(C.Structure):
    _fields_ = [("kind", C.c_int32), ("device", C.c_int32), ("stream", C.c_int32), ("level", C.c_int32),
                ("kernel", C.c_int32), ("group", C.c_int32), ("chunk", C.c_int32), ("nvps", C.c_int32),
                ("bytes", C.c_uint64), ("flops", C.c_double), ("est_ns", C.c_double),
                ("sim_start_ns", C.c_double), ("sim_end_ns", C.c_double), ("measured_ns", C.c_double)]


class SvpError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS_NAMES.get(status, status)}: {msg}")
        self.status = status


_lib = None
_lock = threading.Lock()


def load(build_if_stale: bool = True):
    """Load libsvp.so (building it first when sources are newer and nvcc is present)."""
    global _lib
    with _lock:
        if _lib is not None:
            return _lib
        if build_if_stale and not os.environ.get("SVP_LIB"):
            try:
                from . import _build
                if os.path.exists(_build.NVCC):
                    _build.build()
            except Exception as e:  # a failed build must not silently fall back
                raise RuntimeError(f"building libsvp.so failed: {e}") from e
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} is missing: run `python -m paper_conf_dac_jungc15_b200._build`")
        L = C.CDLL(LIB_PATH)
        P = C.POINTER
        vp = C.c_void_p
        L.svp_config_default.argtypes = [P(svp_config)]
        L.svp_config_default.restype = None
        L.svp_init.argtypes = [P(svp_config), P(vp)]
        L.svp_finalize.argtypes = [vp]
        L.svp_last_error.restype = C.c_char_p
        L.svp_abi_version.restype = C.c_int32
        L.svp_register_kernel.argtypes = [vp, C.c_char_p, P(C.c_int32)]
        L.svp_submit.argtypes = [vp, C.c_int32, C.c_int32, C.c_void_p, C.c_size_t, P(svp_buf), C.c_int32,
                                 P(C.c_uint64)]
        L.svp_submit_batch.argtypes = [vp, C.c_int32, P(svp_job_desc), P(C.c_uint64)]
        L.svp_flush.argtypes = [vp]
        L.svp_vp_device.argtypes = [vp, C.c_int32, P(C.c_int32)]
        L.svp_assign_vps.argtypes = [vp, C.c_int32, P(C.c_int32), P(C.c_int32), P(C.c_double), P(C.c_int32)]
        L.svp_lpt_partition.argtypes = [C.c_int32, P(C.c_int32), P(C.c_double), C.c_int32, P(C.c_int32)]
        L.svp_profile.argtypes = [vp, C.c_int32, P(svp_vp_profile)]
        L.svp_reset_profile.argtypes = [vp]
        L.svp_kernel_stats_get.argtypes = [vp, C.c_int32, P(svp_kernel_stats)]
        L.svp_flush_stats_get.argtypes = [vp, P(svp_flush_stats)]
        L.svp_plan_size.argtypes = [vp, P(C.c_int32)]
        L.svp_plan_get.argtypes = [vp, C.c_int32, P(svp_plan_op), P(C.c_int32), C.c_int32]
        L.svp_wait.argtypes = [vp, C.c_uint64, C.c_int32]
        L.svp_start_dispatcher.argtypes = [vp, C.c_int32, C.c_int32]
        L.svp_stop_dispatcher.argtypes = [vp]
        L.svp_ipc_serve.argtypes = [vp, C.c_char_p, C.c_uint64, C.c_int32, P(vp)]
        L.svp_ipc_server_stats.argtypes = [vp, P(C.c_uint64), P(C.c_uint64)]
        L.svp_ipc_shutdown.argtypes = [vp]
        L.svp_ipc_connect.argtypes = [C.c_char_p, P(vp)]
        L.svp_ipc_disconnect.argtypes = [vp]
        L.svp_ipc_alloc.argtypes = [vp, C.c_uint64, P(C.c_uint64), P(vp)]
        L.svp_ipc_submit.argtypes = [vp, C.c_int32, C.c_int32, C.c_void_p, C.c_size_t, P(svp_ipc_buf), C.c_int32,
                                     P(C.c_uint64)]
        L.svp_ipc_wait.argtypes = [vp, C.c_uint64, C.c_int32]
        L.svp_kernel_lookup.argtypes = [C.c_char_p, P(C.c_int32)]
        L.svp_device_stats_get.argtypes = [vp, C.c_int32, P(svp_device_stats)]
        L.svp_host_alloc.argtypes = [vp, C.c_int32, C.c_uint64, P(C.c_void_p), P(C.c_int32)]
        L.svp_host_free.argtypes = [vp, C.c_void_p]
        L.svp_flush_async.argtypes = [vp, P(C.c_uint64)]
        L.svp_flush_wait.argtypes = [vp, C.c_uint64]
        L.svp_plan_op_detail.argtypes = [vp, C.c_int32, P(C.c_uint64), P(C.c_uint64), P(C.c_int32), C.c_int32,
                                         P(C.c_int32), P(C.c_double)]
        for name in EXPORTS:
            f = getattr(L, name)
            if name not in ("svp_config_default", "svp_last_error", "svp_abi_version"):
                f.restype = C.c_int32
        _lib = L
    return _lib


def last_error() -> str:
    return load().svp_last_error().decode()


def _check(st: int):
    if st != SVP_OK:
        raise SvpError(st, last_error())


# ----------------------------------------------------------------- argument blobs
def args_vecadd(n: int) -> bytes:
    return struct.pack("<Q", n)


def args_saxpy(n: int, a: float) -> bytes:
    return struct.pack("<QfI", n, a, 0)


def args_hist256(n: int) -> bytes:
    return struct.pack("<Q", n)


def args_blackscholes(n: int, R: float, V: float) -> bytes:
    return struct.pack("<Qff", n, R, V)


def args_sgemm(M: int, N: int, K: int, alpha: float = 1.0, beta: float = 0.0) -> bytes:
    return struct.pack("<iiiff", M, N, K, alpha, beta)


def args_dgemm(M: int, N: int, K: int, alpha: float = 1.0, beta: float = 0.0) -> bytes:
    return struct.pack("<iiiidd", M, N, K, 0, alpha, beta)


Buf = Tuple[int, int, int, int]  # (ptr, bytes, dir, mem)


def lpt_partition(classes: Sequence[int], costs: Sequence[float], G: int) -> List[int]:
    L = load()
    n = len(classes)
    cl = (C.c_int32 * n)(*classes)
    co = (C.c_double * n)(*costs)
    out = (C.c_int32 * n)()
    _check(L.svp_lpt_partition(n, cl, co, G, out))
    return list(out)


class JobBatch:
    """A pre-marshalled svp_job_desc array: build once, submit many times (a VP that
    resubmits the same kernel on the same buffers pays no Python marshalling)."""

    def __init__(self, jobs: Sequence[Tuple[int, int, bytes, Sequence[Buf]]]):
        self.n = len(jobs)
        self.arr = (svp_job_desc * max(1, self.n))()
        for i, (vp, kid, args, bufs) in enumerate(jobs):
            d = self.arr[i]
            d.vp, d.kernel, d.args_bytes, d.nbufs = vp, kid, len(args), len(bufs)
            C.memmove(d.args, args, len(args))
            for b, (p, nb, dr, m) in enumerate(bufs):
                d.bufs[b] = svp_buf(p, nb, dr, m)
        self.ids = (C.c_uint64 * max(1, self.n))()


class Context:
    """Owns one svp_ctx.  Keyword arguments mirror svp_config fields."""

    def __init__(self, num_gpus: int = 0, device_ids: Optional[Sequence[int]] = None, streams_per_gpu: int = 4,
                 coalesce: bool = True, interleave: bool = True, max_chunks: int = 8, arena_bytes: int = 0,
                 profile_level: int = 0, sync_each_job: bool = False, dry_run: bool = False,
                 flush_timeout_ms: int = 0, validate_ptrs: int = 1, sgemm_impl: int = SGEMM_TF32BF16,
                 external_streams: Optional[Sequence[int]] = None, hbm_gbps: float = 0.0, pcie_gbps: float = 0.0,
                 ffma_tflops: float = 0.0, launch_us: float = 0.0, hetero: bool = False, graph: bool = True,
                 table_mode: int = TABLE_PARAM, sgemm_kchunk: Optional[int] = None):
        L = load()
        cfg = svp_config()
        L.svp_config_default(C.byref(cfg))
        cfg.num_gpus = num_gpus
        self._ids = None
        if device_ids is not None:
            self._ids = (C.c_int32 * len(device_ids))(*device_ids)
            cfg.device_ids = C.cast(self._ids, C.POINTER(C.c_int32))
            cfg.num_gpus = len(device_ids)
        cfg.streams_per_gpu = streams_per_gpu
        cfg.coalesce = int(coalesce)
        cfg.interleave = int(interleave)
        cfg.max_chunks = max_chunks
        cfg.arena_bytes = arena_bytes
        cfg.profile_level = profile_level
        cfg.sync_each_job = int(sync_each_job)
        cfg.dry_run = int(dry_run)
        cfg.flush_timeout_ms = flush_timeout_ms
        cfg.validate_ptrs = int(validate_ptrs)
        cfg.sgemm_impl = int(sgemm_impl)
        self._ext = None
        if external_streams is not None:
            self._ext = (C.c_void_p * len(external_streams))(*external_streams)
            cfg.external_streams = C.cast(self._ext, C.POINTER(C.c_void_p))
        cfg.hbm_gbps, cfg.pcie_gbps, cfg.ffma_tflops, cfg.launch_us = hbm_gbps, pcie_gbps, ffma_tflops, launch_us
        cfg.hetero, cfg.graph, cfg.table_mode = int(hetero), int(graph), int(table_mode)
        if sgemm_kchunk is not None:  # else the library default (svp_config_default)
            cfg.sgemm_kchunk = int(sgemm_kchunk)
        h = C.c_void_p()
        _check(L.svp_init(C.byref(cfg), C.byref(h)))
        self._h = h
        self._L = L
        self.kernel_ids: Dict[str, int] = {}

    # -------------------------------------------------------------- lifetime
    def close(self):
        if getattr(self, "_h", None):
            _check(self._L.svp_finalize(self._h))
            self._h = None

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # -------------------------------------------------------------- API
    def register_kernel(self, name: str) -> int:
        kid = C.c_int32()
        _check(self._L.svp_register_kernel(self._h, name.encode(), C.byref(kid)))
        self.kernel_ids[name] = kid.value
        return kid.value

    def kernel(self, name: str) -> int:
        return self.kernel_ids.get(name) or self.register_kernel(name)

    def submit(self, vp: int, kernel: int, args: bytes, bufs: Sequence[Buf]) -> int:
        arr = (svp_buf * max(1, len(bufs)))(*[svp_buf(p, b, d, m) for (p, b, d, m) in bufs])
        jid = C.c_uint64()
        ab = C.create_string_buffer(args, len(args))
        _check(self._L.svp_submit(self._h, vp, kernel, ab, len(args), arr, len(bufs), C.byref(jid)))
        return jid.value

    def submit_batch(self, jobs) -> List[int]:
        """jobs: a JobBatch, or a sequence of (vp, kernel id, args, bufs)."""
        if isinstance(jobs, JobBatch):
            _check(self._L.svp_submit_batch(self._h, jobs.n, jobs.arr, jobs.ids))
            return jobs.ids
        n = len(jobs)
        arr = (svp_job_desc * max(1, n))()
        for i, (vp, kid, args, bufs) in enumerate(jobs):
            d = arr[i]
            d.vp, d.kernel, d.args_bytes, d.nbufs = vp, kid, len(args), len(bufs)
            C.memmove(d.args, args, len(args))
            for b, (p, nb, dr, m) in enumerate(bufs):
                d.bufs[b] = svp_buf(p, nb, dr, m)
        ids = (C.c_uint64 * max(1, n))()
        _check(self._L.svp_submit_batch(self._h, n, arr, ids))
        return list(ids)[:n]

    def flush(self):
        _check(self._L.svp_flush(self._h))

    def flush_async(self) -> int:
        """svp_flush_async: enqueue the flush and return its ticket; it completes when the
        next flush has been issued, or at flush_wait(ticket)."""
        t = C.c_uint64()
        _check(self._L.svp_flush_async(self._h, C.byref(t)))
        return t.value

    def flush_wait(self, ticket: int):
        _check(self._L.svp_flush_wait(self._h, ticket))

    def wait(self, job: int, timeout_ms: int = 0):
        """VP Control: block until `job` has run (svp_wait).  Releases the GIL."""
        _check(self._L.svp_wait(self._h, job, timeout_ms))

    def start_dispatcher(self, window_us: int = 50, max_jobs: int = 0):
        _check(self._L.svp_start_dispatcher(self._h, window_us, max_jobs))

    def stop_dispatcher(self):
        _check(self._L.svp_stop_dispatcher(self._h))

    def vp_device(self, vp: int) -> int:
        d = C.c_int32()
        _check(self._L.svp_vp_device(self._h, vp, C.byref(d)))
        return d.value

    def assign_vps(self, vps: Sequence[int], classes: Sequence[int], costs: Sequence[float]) -> List[int]:
        n = len(vps)
        out = (C.c_int32 * max(1, n))()
        _check(self._L.svp_assign_vps(self._h, n, (C.c_int32 * max(1, n))(*vps), (C.c_int32 * max(1, n))(*classes),
                                      (C.c_double * max(1, n))(*costs), out))
        return list(out)[:n]

    def profile(self, vp: int = -1) -> Dict[str, float]:
        p = svp_vp_profile()
        _check(self._L.svp_profile(self._h, vp, C.byref(p)))
        return {k: getattr(p, k) for k, _ in svp_vp_profile._fields_}

    def reset_profile(self):
        _check(self._L.svp_reset_profile(self._h))

    def kernel_stats(self, kernel: int) -> Dict[str, float]:
        s = svp_kernel_stats()
        _check(self._L.svp_kernel_stats_get(self._h, kernel, C.byref(s)))
        return {k: getattr(s, k) for k, _ in svp_kernel_stats._fields_}

    def device_stats(self, g: int) -> Dict[str, float]:
        s = svp_device_stats()
        _check(self._L.svp_device_stats_get(self._h, g, C.byref(s)))
        return {k: getattr(s, k) for k, _ in svp_device_stats._fields_}

    def host_alloc(self, gpu: int, nbytes: int):
        """svp_host_alloc: page-locked host memory on GPU index `gpu`'s NUMA node.
        Returns (address, numa node or -1)."""
        p, node = C.c_void_p(), C.c_int32()
        _check(self._L.svp_host_alloc(self._h, gpu, nbytes, C.byref(p), C.byref(node)))
        return p.value, node.value

    def host_free(self, addr: int):
        _check(self._L.svp_host_free(self._h, addr))

    def flush_stats(self) -> Dict[str, float]:
        s = svp_flush_stats()
        _check(self._L.svp_flush_stats_get(self._h, C.byref(s)))
        return {k: getattr(s, k) for k, _ in svp_flush_stats._fields_}

    def plan(self) -> List[Dict]:
        n = C.c_int32()
        _check(self._L.svp_plan_size(self._h, C.byref(n)))
        out = []
        for i in range(n.value):
            op = svp_plan_op()
            vps = (C.c_int32 * 4096)()
            _check(self._L.svp_plan_get(self._h, i, C.byref(op), vps, 4096))
            d = {k: getattr(op, k) for k, _ in svp_plan_op._fields_}
            d["vps"] = list(vps[: min(op.nvps, 4096)])
            aoff, alen, nw, t0 = C.c_uint64(), C.c_uint64(), C.c_int32(), C.c_double()
            waits = (C.c_int32 * 256)()
            _check(self._L.svp_plan_op_detail(self._h, i, C.byref(aoff), C.byref(alen), waits, 256, C.byref(nw),
                                              C.byref(t0)))
            d["arena_off"], d["arena_len"], d["measured_start_ns"] = aoff.value, alen.value, t0.value
            d["waits"] = list(waits[: min(nw.value, 256)])
            out.append(d)
        return out


# ----------------------------------------------------------------- IPC front end
def kernel_lookup(name: str) -> int:
    kid = C.c_int32()
    _check(load().svp_kernel_lookup(name.encode(), C.byref(kid)))
    return kid.value


class IpcServer:
    """svp_ipc_serve: serve VP processes through the shared-memory segment `name`."""

    def __init__(self, ctx: "Context", name: str, arena_bytes: int = 1 << 28, nslots: int = 1024):
        self._L = load()
        h = C.c_void_p()
        _check(self._L.svp_ipc_serve(ctx._h, name.encode(), arena_bytes, nslots, C.byref(h)))
        self._h = h
        self.ctx = ctx

    def stats(self):
        served, tickets = C.c_uint64(), C.c_uint64()
        _check(self._L.svp_ipc_server_stats(self._h, C.byref(served), C.byref(tickets)))
        return {"served": served.value, "tickets": tickets.value}

    def shutdown(self):
        if getattr(self, "_h", None):
            _check(self._L.svp_ipc_shutdown(self._h))
            self._h = None

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.shutdown()


class IpcClient:
    """A VP process's view of an IpcServer (no CUDA needed in this process)."""

    def __init__(self, name: str):
        self._L = load(build_if_stale=False)
        h = C.c_void_p()
        _check(self._L.svp_ipc_connect(name.encode(), C.byref(h)))
        self._h = h

    def alloc(self, nbytes: int):
        """Returns (offset, address) of nbytes in the shared arena."""
        off, ptr = C.c_uint64(), C.c_void_p()
        _check(self._L.svp_ipc_alloc(self._h, nbytes, C.byref(off), C.byref(ptr)))
        return off.value, ptr.value

    def submit(self, vp: int, kernel: int, args: bytes, bufs: Sequence[Tuple[int, int, int]]) -> int:
        """bufs: (arena offset, bytes, dir).  Returns a ticket."""
        arr = (svp_ipc_buf * max(1, len(bufs)))(*[svp_ipc_buf(o, b, d, 0) for (o, b, d) in bufs])
        t = C.c_uint64()
        ab = C.create_string_buffer(args, len(args))
        _check(self._L.svp_ipc_submit(self._h, vp, kernel, ab, len(args), arr, len(bufs), C.byref(t)))
        return t.value

    def wait(self, ticket: int, timeout_ms: int = 0):
        _check(self._L.svp_ipc_wait(self._h, ticket, timeout_ms))

    def close(self):
        if getattr(self, "_h", None):
            _check(self._L.svp_ipc_disconnect(self._h))
            self._h = None
