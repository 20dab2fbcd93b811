"""VP buffer sets: allocate each VP's buffers with PyTorch and marshal them into jobs.

PyTorch is only the allocator here (device memory or page-locked host memory); the
job descriptors go straight to :class:`svp.Context` and everything that computes runs
in libsvp.so.  A "spec" is any object with the attributes ``vp, kernel, n, M, N, K, a,
R, V, alpha, beta, misalign`` (see workloads.JobSpec); inputs are numpy arrays keyed by
buffer name.  Every buffer is followed by a 64-byte guard of 0xAB so tests can check
that no kernel wrote past a VP's extent (the segment table needs no padding).
"""
from __future__ import annotations

import ctypes
from typing import Dict, List, Optional, Sequence

import numpy as np
import torch

from . import svp

BUFS = {
    "vecadd": [("a", "f32", svp.DIR_IN), ("b", "f32", svp.DIR_IN), ("c", "f32", svp.DIR_OUT)],
    "saxpy": [("x", "f32", svp.DIR_IN), ("y", "f32", svp.DIR_INOUT)],
    "hist256": [("d", "u8", svp.DIR_IN), ("counts", "u32", svp.DIR_OUT)],
    "blackscholes": [("S", "f32", svp.DIR_IN), ("X", "f32", svp.DIR_IN), ("T", "f32", svp.DIR_IN),
                     ("call", "f32", svp.DIR_OUT), ("put", "f32", svp.DIR_OUT)],
    "sgemm": [("A", "f32", svp.DIR_IN), ("B", "f32", svp.DIR_IN), ("C", "f32", svp.DIR_OUT)],
    "sgemm_tf32": [("A", "f32", svp.DIR_IN), ("B", "f32", svp.DIR_IN), ("C", "f32", svp.DIR_OUT)],
    "dgemm": [("A", "f64", svp.DIR_IN), ("B", "f64", svp.DIR_IN), ("C", "f64", svp.DIR_OUT)],
}
GEMMS = ("sgemm", "sgemm_tf32", "dgemm")
_TORCH = {"f32": torch.float32, "u8": torch.uint8, "u32": torch.int32, "f64": torch.float64}
_NP = {"f32": np.float32, "u8": np.uint8, "u32": np.uint32, "f64": np.float64}
_ES = {"f32": 4, "u8": 1, "u32": 4, "f64": 8}
GUARD = 64


def buffer_elems(spec, name: str) -> int:
    k = spec.kernel
    if k in GEMMS:
        return {"A": spec.M * spec.K, "B": spec.K * spec.N, "C": spec.M * spec.N}[name]
    if k == "hist256" and name == "counts":
        return 256
    return spec.n


def job_args(spec) -> bytes:
    k = spec.kernel
    if k == "vecadd":
        return svp.args_vecadd(spec.n)
    if k == "saxpy":
        return svp.args_saxpy(spec.n, spec.a)
    if k == "hist256":
        return svp.args_hist256(spec.n)
    if k == "blackscholes":
        return svp.args_blackscholes(spec.n, spec.R, spec.V)
    if k == "dgemm":
        return svp.args_dgemm(spec.M, spec.N, spec.K, spec.alpha, spec.beta)
    return svp.args_sgemm(spec.M, spec.N, spec.K, spec.alpha, spec.beta)


class VPSet:
    """Buffers of a list of jobs, resident on the VP's GPU ("device") or pinned host ("host")."""

    def __init__(self, ctx: svp.Context, specs: Sequence, inputs: Optional[Sequence[Dict[str, np.ndarray]]] = None,
                 residency: str = "device", device_ordinals: Optional[Sequence[int]] = None,
                 assign: bool = True, host_numa: bool = False):
        """host_numa (residency "host"): allocate every VP's buffers with svp_host_alloc on the
        NUMA node of the GPU the Dispatcher placed the VP on (the VPs are assigned first)."""
        self.ctx = ctx
        self.specs = list(specs)
        self.residency = residency
        self.kids = {}
        for s in self.specs:
            if s.kernel not in self.kids:
                self.kids[s.kernel] = ctx.kernel(s.kernel)
        self.host_blocks: List[int] = []
        if assign and (residency == "device" or host_numa):
            self.assign_to(ctx)
        self.bufs: List[Dict[str, torch.Tensor]] = []   # views (what the kernel sees)
        self.raw: List[Dict[str, torch.Tensor]] = []    # allocations incl. misalign + guard
        self.offsets: List[Dict[str, int]] = []
        for i, s in enumerate(self.specs):
            if residency == "device":
                g = ctx.vp_device(s.vp)
                dev = torch.device("cuda", device_ordinals[g] if device_ordinals else g)
            else:
                dev = torch.device("cpu")
            views, raws, offs = {}, {}, {}
            m = getattr(s, "misalign", 0)
            for bi, (name, dt, _dir) in enumerate(BUFS[s.kernel]):
                ne = buffer_elems(s, name)
                es = _ES[dt]
                # misalign 1: every buffer shifted by one element (co-aligned -> vector path
                # with a head shift); misalign 2: only the first buffer (scalar path)
                mis = m if (m == 1 or bi == 0) else 0
                if s.kernel in GEMMS:
                    mis = m  # every matrix shifted by m elements (m = 1: 4-B offset, not 16-B aligned)
                elif s.kernel == "hist256" and name == "counts":
                    mis = 0
                elif s.kernel == "hist256":
                    mis = 7 * m
                nbytes = (ne + mis) * es + GUARD
                if dev.type == "cpu" and host_numa:
                    addr, _node = ctx.host_alloc(ctx.vp_device(s.vp), nbytes)
                    self.host_blocks.append(addr)
                    raw = torch.frombuffer((ctypes.c_uint8 * nbytes).from_address(addr), dtype=torch.uint8)
                elif dev.type == "cpu":
                    raw = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
                else:
                    raw = torch.empty(nbytes, dtype=torch.uint8, device=dev)
                raw[(ne + mis) * es:].fill_(0xAB)
                view = raw[mis * es: (ne + mis) * es].view(_TORCH[dt])
                views[name], raws[name], offs[name] = view, raw, mis * es
            self.bufs.append(views)
            self.raw.append(raws)
            self.offsets.append(offs)
        self.inputs = inputs
        if inputs is not None:
            self.load_inputs()

    def assign_to(self, ctx: svp.Context):
        """Register this set's kernels in ctx and pin its VPs to GPUs with the Dispatcher's
        kernel-stratified LPT (deterministic: a second context sharing these buffers gets
        the same placement)."""
        for name in self.kids:
            ctx.kernel(name)
        # estimated kernel ns (the Dispatcher's LPT costs): algorithmic bytes at the measured
        # 6.55 TB/s (6550 B/ns) + FLOPs at ~400 TFLOP/s (4e5 flop/ns, the fp32 tensor-core split)
        costs = [float(s.algorithmic_bytes()) / 6550.0 + float(s.flops()) / 4.0e5 for s in self.specs]
        ctx.assign_vps([s.vp for s in self.specs], [self.kids[s.kernel] for s in self.specs], costs)

    def release_host(self):
        """svp_host_free every host_numa block (else the context frees them at close).  The
        buffer views must not be used afterwards."""
        for a in self.host_blocks:
            self.ctx.host_free(a)
        self.host_blocks = []
        self.bufs, self.raw = [], []

    def load_inputs(self):
        for i, s in enumerate(self.specs):
            inp = self.inputs[i]
            for name, dt, d in BUFS[s.kernel]:
                if s.kernel in GEMMS and name == "C" and s.beta != 0:
                    d = svp.DIR_INOUT  # C is read when beta != 0
                if d & svp.DIR_IN and name in inp:
                    src = torch.from_numpy(np.ascontiguousarray(inp[name]).reshape(-1).view(_NP[dt]))
                    if dt == "u32":
                        src = src.view(torch.int32)
                    self.bufs[i][name].copy_(src, non_blocking=False)
                elif not (d & svp.DIR_IN):
                    # outputs start as NaN/garbage so a missing write is caught
                    v = self.bufs[i][name]
                    if v.numel():
                        if v.dtype in (torch.float32, torch.float64):
                            v.fill_(float("nan"))
                        else:
                            v.fill_(-1 if v.dtype == torch.int32 else 0x5A)

    def job_list(self):
        jobs = []
        for i, s in enumerate(self.specs):
            mem = svp.MEM_HOST_PINNED if self.residency == "host" else svp.MEM_DEVICE
            bl = []
            for name, dt, d in BUFS[s.kernel]:
                t = self.bufs[i][name]
                if s.kernel in GEMMS and name == "C" and s.beta != 0:
                    d = svp.DIR_INOUT
                bl.append((t.data_ptr() if t.numel() else 0, t.numel() * t.element_size(), d, mem))
            jobs.append((s.vp, self.kids[s.kernel], job_args(s), bl))
        return jobs

    def submit(self) -> List[int]:
        return self.ctx.submit_batch(self.job_list())

    def output(self, i: int) -> Dict[str, np.ndarray]:
        s = self.specs[i]
        out = {}
        for name, dt, d in BUFS[s.kernel]:
            if d & svp.DIR_OUT or (s.kernel in GEMMS and name == "C"):
                t = self.bufs[i][name].cpu()
                a = t.numpy()
                if dt == "u32":
                    a = a.view(np.uint32)
                if s.kernel in GEMMS:
                    a = a.reshape(s.M, s.N)
                out[name] = a.copy()
        return out

    def guards_intact(self) -> bool:
        for i, s in enumerate(self.specs):
            for name, dt, _ in BUFS[s.kernel]:
                raw = self.raw[i][name]
                g = raw[raw.numel() - GUARD:].cpu()
                if not bool((g == 0xAB).all()):
                    return False
        return True
