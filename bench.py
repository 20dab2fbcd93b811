#!/usr/bin/env python
"""bench.py -- ΣVP hot path on B200: VP-kernel jobs/s (+ HBM GB/s, speedup vs serial launch).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl svp|reference] [--config 5]

A *step* is one pass of the whole hot path over one batch: every VP of the workload
submits its job (svp_submit_batch -> Job Queue), then svp_flush runs Kernel Match ->
Job Dispatcher -> Re-scheduler -> coalesced sm_100a kernels (interleaved streams) ->
Profiler and returns when every output is in place.  Default workload = BASELINE.json
config 5 (256 VPs: vecadd/SAXPY/hist256/Black-Scholes with ragged 64Ki-16Mi sizes +
SGEMM 2048^3), the configuration the north-star target is stated on.  At N GPUs
(`--scaling weak`, the default) the workload is N x 256 independent VPs and the Job
Dispatcher's kernel-stratified LPT partition shards them over the ranks, 256 per GPU
(no data-path collective: VPs share no data); `--scaling strong` splits the fixed 256.

`value` is device-timed (CUDA events on the stream the library joins, max over ranks)
with every VP's buffers resident in HBM; `e2e` is the same metric with pinned HOST
buffers (H2D + D2H inside the timed region, Kernel Interleaving on).  The working set
(~9 GB) is far larger than L2, so no L2 flush is needed between steps.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import workloads as W  # noqa: E402

METRIC = "VP-kernel jobs/sec & HBM GB/s vs #VPs at 1/2/4/8 B200; speedup vs serial launch"
CONFIG_NAMES = {
    1: "cfg1: 2 VPs x vecadd 1Mi",
    2: "cfg2: 16 VPs x SGEMM 512^3 fp32",
    3: "cfg3: 64 VPs mixed vecadd/SAXPY/hist256/Black-Scholes 4Mi",
    4: "cfg4: 64 VPs mixed, ragged 64Ki-16Mi + adversarial sizes",
    5: "cfg5: 256 VPs mixed vecadd/SAXPY/hist256/Black-Scholes (ragged 64Ki-16Mi) + SGEMM 2048^3",
}


IMPL_NAMES = ("ffma", "3xtf32", "tf32bf16")  # svp.SGEMM_FFMA, SGEMM_3XTF32, SGEMM_TF32BF16
IMPLS = {n: i for i, n in enumerate(IMPL_NAMES)}
# what the path computes in: the memory-bound kernels are fp32 (u8 -> u32 for hist256); the
# fp32 "sgemm" contract (1e-5) is met by the selected implementation
DTYPE_LABEL = {"tf32bf16": "f32 (sgemm: tf32 + 2x bf16 MMAs on an operand hi/lo split, f32 accumulate)",
               "3xtf32": "f32 (sgemm: 3x tf32 MMAs on an operand hi/lo split, f32 accumulate)",
               "ffma": "f32"}


# ----------------------------------------------------------------------------- helpers
def trace(msg):
    if os.environ.get("SVP_BENCH_TRACE"):
        print(f"[rank {os.environ.get('RANK', '0')}] {time.strftime('%H:%M:%S')} {msg}", file=sys.stderr, flush=True)


def dist_setup():
    """One process per GPU (torchrun).  SVP_BENCH_DEVICE=<ordinal> pins every rank to one
    GPU (tests the multi-rank path on a 1-GPU box).  The process group is gloo: it only
    carries the barrier and the max / sum of a few timing scalars -- the data path has no
    collective (VPs share no data; BASELINE.json: "NCCL is not used")."""
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    forced = os.environ.get("SVP_BENCH_DEVICE")
    if forced is not None:
        local = int(forced)
    if ws > 1:
        import torch.distributed as dist
        import torch
        if torch.cuda.is_available():
            torch.cuda.set_device(local)
        dist.init_process_group(backend="gloo")
    return rank, ws, local


def barrier(ws):
    if ws > 1:
        import torch.distributed as dist
        dist.barrier()


def max_over_ranks(x: float, ws: int) -> float:
    if ws == 1:
        return x
    import torch
    import torch.distributed as dist
    t = torch.tensor([x], dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def sum_over_ranks(x: float, ws: int) -> float:
    if ws == 1:
        return x
    import torch
    import torch.distributed as dist
    t = torch.tensor([x], dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.SUM)
    return float(t.item())


def my_specs(specs, rank, ws):
    """Job Dispatcher across ranks: the same kernel-stratified LPT every rank computes."""
    if ws == 1:
        return list(specs)
    from paper_conf_dac_jungc15_b200 import svp
    classes = [W.KERNELS.index(s.kernel) for s in specs]
    costs = [s.algorithmic_bytes() / 6.5e12 + s.flops() / 60e12 for s in specs]
    part = svp.lpt_partition(classes, costs, ws)
    return [s for s, p in zip(specs, part) if p == rank]


class Clocks:
    """nvidia-smi sampling of the timed region (B200_PROFILING.md clocks line).

    The sampler starts before the warm-up (nvidia-smi takes ~0.1-0.3 s to emit its first
    line, longer than a short timed region), stamps every sample, and `stop()` keeps the
    samples whose timestamps fall inside [mark_start(), mark_end()]; if fewer than 3 do,
    the nearest samples around the window are added and `in_window` says how many were
    strictly inside."""

    # power.draw.instant: plain power.draw is a 1-s average on Ampere and newer, which
    # mostly shows the idle time before a ~0.1-s timed region
    Q = ("timestamp,index,clocks.sm,clocks.max.sm,power.draw.instant,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap,enforced.power.limit")

    def __init__(self, device_indices):
        self.p = None
        self.t0 = self.t1 = None
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        if isinstance(device_indices, int):
            device_indices = [device_indices]
        try:
            import torch
            uu = []
            for d in device_indices:
                u = str(torch.cuda.get_device_properties(d).uuid)
                uu.append(u if u.startswith("GPU-") else "GPU-" + u)
            ident = ["--id=" + ",".join(uu)] if uu else []
        except Exception:
            ident = []
        try:
            self.p = subprocess.Popen(["nvidia-smi"] + ident + ["--query-gpu=" + self.Q, "--format=csv,noheader,nounits",
                                                                 "-lms", "20"], stdout=self.f, stderr=subprocess.DEVNULL)
            deadline = time.time() + 5.0
            while time.time() < deadline and os.path.getsize(self.f.name) == 0:
                time.sleep(0.02)
        except Exception:
            self.p = None

    def mark_start(self):
        self.t0 = time.time()

    def mark_end(self):
        self.t1 = time.time()

    @staticmethod
    def _ts(text):
        import datetime
        try:
            return datetime.datetime.strptime(text.strip(), "%Y/%m/%d %H:%M:%S.%f").timestamp()
        except ValueError:
            return None

    def stop(self):
        if self.p is None:
            return None
        time.sleep(0.1)
        self.p.terminate()
        try:
            self.p.wait(timeout=5)
        except Exception:
            self.p.kill()
        self.f.flush()
        self.f.seek(0)
        rows = []
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in self.f.read().splitlines():
            parts = [x.strip() for x in line.split(",")]
            if len(parts) < 10:
                continue
            try:
                pw = float(parts[4]) if parts[4] not in ("", "[N/A]") else float("nan")
                try:
                    lim = float(parts[10]) if len(parts) > 10 else float("nan")
                except ValueError:
                    lim = float("nan")
                rows.append((self._ts(parts[0]), float(parts[2]), float(parts[3]), parts[6:10], pw, lim))
            except ValueError:
                continue
        os.unlink(self.f.name)
        rows = [r for r in rows if r[0] is not None]
        if not rows or self.t0 is None or self.t1 is None:
            return None
        inside = [r for r in rows if self.t0 <= r[0] <= self.t1]
        sel = list(inside)
        if len(sel) < 3:  # short window: add the samples nearest to it
            mid = 0.5 * (self.t0 + self.t1)
            sel = sorted(rows, key=lambda r: abs(r[0] - mid))[:3]
        reasons = set()
        for r in sel:
            for nm, val in zip(names, r[3]):
                if val.lower().startswith("active"):
                    reasons.add(nm)
        pws = [r[4] for r in sel if r[4] == r[4]]
        lims = [r[5] for r in sel if r[5] == r[5]]
        return {"sm_mhz": statistics.median(r[1] for r in sel), "sm_max_mhz": max(r[2] for r in sel),
                "samples": len(sel), "in_window": len(inside), "window_ms": (self.t1 - self.t0) * 1e3,
                "reasons": sorted(reasons), "power_w": statistics.median(pws) if pws else None,
                "power_field": "power.draw.instant (median of the samples)",
                "power_limit_w": statistics.median(lims) if lims else None}


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            return json.load(f), "measured"
    return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "sm_max_mhz": 1965.0}, "fallback"


def cpu_baseline(specs, inputs, label):
    """The oracle as it stands on the host cores: a proportional sample of the workload
    (the first min(#VPs, 5 x cores) VPs -- VP v runs kernel v % 5, so every class keeps
    its share), each VP single-threaded, VPs spread over the cores."""
    import oracle
    cores = len(os.sched_getaffinity(0))
    n = min(len(specs), 5 * cores)
    sp, inp = specs[:n], inputs[:n]
    oracle.build()
    t0 = time.perf_counter()
    oracle.run_jobs(sp, inp, threads=cores)
    dt = time.perf_counter() - t0
    kinds = {}
    for s in sp:
        kinds[s.kernel] = kinds.get(s.kernel, 0) + 1
    return {"value": n / dt, "unit": "jobs/s", "cores": min(cores, n), "kind": "oracle",
            "sample": f"{n} of {len(specs)} VPs of {label} ({', '.join(f'{v} {k}' for k, v in kinds.items())}), "
                      f"one oracle pass, wall {dt:.2f} s"}


# ----------------------------------------------------------------------------- arms
def run_reference(args, rank, ws):
    """--impl reference: the oracle (the paper's emulation baseline) on host cores."""
    if rank != 0:
        return
    specs = W.config_specs(args.config, nvps=args.vps)
    cores = len(os.sched_getaffinity(0))
    # bounded sample: the first n VPs (kernel = vp % 5 keeps every class's share), n sized
    # so (warmup + steps) passes take about 2-3 minutes on this box's cores
    n = min(len(specs), 5 * cores)
    if args.steps + args.warmup > 33:
        n = max(5, (n * 33 // (args.steps + args.warmup)) // 5 * 5)
    sample = specs[:n]
    inputs = W.make_inputs_many(sample)
    import oracle
    oracle.build()
    for _ in range(args.warmup):
        oracle.run_jobs(sample, inputs, threads=cores)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        oracle.run_jobs(sample, inputs, threads=cores)
    dt = time.perf_counter() - t0
    value = n * args.steps / dt
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": "jobs/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt / args.steps * 1e3,
            "higher_is_better": True, "scaling": "strong" if args.gpus > 1 else "weak", "vs_baseline": None,
            "dtype": "f64 accumulation for sgemm (oracle), f32 elsewhere", "data": "synthetic",
            "config": {"workload": CONFIG_NAMES[args.config], "config_index": args.config, "vps": len(specs),
                       "sample_vps": n,
                       "parallelism": f"host threads x{min(cores, n)}"},
            "cpu_baseline": {"value": value, "unit": "jobs/s", "cores": min(cores, n), "kind": "oracle",
                             "sample": f"first {n} of {len(specs)} VPs (kernel = vp % 5) per step"},
            "e2e": {"value": value, "unit": "jobs/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


L2_BYTES = 126 << 20  # B200 L2 (B200_PROFILING.md)


def n_buffer_sets(specs):
    """Rotating buffer sets so that consecutive steps never find their inputs in L2: one set
    when a step's working set is already >= 4 x L2, else enough sets to cover 4 x L2
    (cfg1: 24 MiB per step -> 24 sets; cfg2: 48 MiB -> 11 sets)."""
    ws = sum(s.input_bytes() + s.output_bytes() for s in specs)
    return 1 if ws >= 4 * L2_BYTES else -(-4 * L2_BYTES // max(1, ws))


def l2_note(specs, nsets):
    ws = sum(s.input_bytes() + s.output_bytes() for s in specs)
    if nsets == 1:
        return "inputs > L2: %.2f GB of VP buffers touched per step" % (ws / 1e9)
    return ("step working set %.1f MiB < L2: %d rotating buffer sets (%.0f MiB > 4 x L2), step i uses set i mod %d"
            % (ws / 2**20, nsets, nsets * ws / 2**20, nsets))


class Arm:
    """One svp.Context driving this process's GPUs, and the workload's VP buffers (one or
    more rotating buffer sets) pre-marshalled as JobBatches."""

    def __init__(self, specs, inputs, residency, ordinals, streams, nsets=1, kids=None, host_numa=False,
                 share=None, async_flush=False, **cfg):
        """share: another device-resident Arm whose buffer sets (and job batches) this one
        reuses -- its VPs are placed on the same GPUs by the same deterministic LPT."""
        from paper_conf_dac_jungc15_b200 import svp
        from paper_conf_dac_jungc15_b200.vpset import VPSet
        self.svp = svp
        self.async_flush = async_flush
        self.ticket = 0
        self.ordinals = list(ordinals)
        self.streams = streams
        self.ctx = svp.Context(num_gpus=len(self.ordinals), device_ids=self.ordinals,
                               external_streams=[st.cuda_stream for st in streams], **cfg)
        if share is not None:
            share.sets[0].assign_to(self.ctx)
            self.sets, self.batches = share.sets, share.batches
        else:
            self.sets = [VPSet(self.ctx, specs, inputs, residency,
                               device_ordinals=self.ordinals if residency == "device" else None,
                               host_numa=host_numa)
                         for _ in range(nsets)]
            self.batches = [svp.JobBatch(vs.job_list()) for vs in self.sets]
        self.kids = self.sets[0].kids
        self.i = 0

    def step(self):
        self.ctx.submit_batch(self.batches[self.i % len(self.batches)])
        if self.async_flush:
            self.ticket = self.ctx.flush_async()
        else:
            self.ctx.flush()
        self.i += 1

    def steps(self, k):
        """k steps; with async flushes (svp_flush_async) step i's device work overlaps step
        i+1's submit / plan / issue, and the last step is completed (svp_flush_wait) before
        returning, so k steps means k completed flushes."""
        for _ in range(k):
            self.step()
        if self.async_flush and self.ticket:
            self.ctx.flush_wait(self.ticket)

    def timed(self, k):
        """k steps bracketed by CUDA events on every GPU's stream (the stream the library
        joins); returns (max over GPUs, per-GPU seconds)."""
        import torch
        evs = []
        for d, st in zip(self.ordinals, self.streams):
            torch.cuda.synchronize(d)
        for st in self.streams:
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(st)
            evs.append((e0, e1))
        self.steps(k)
        for (e0, e1), st in zip(evs, self.streams):
            e1.record(st)
        for d in set(self.ordinals):
            torch.cuda.synchronize(d)
        per = [e0.elapsed_time(e1) / 1e3 for e0, e1 in evs]
        return max(per), per

    def device_stats(self):
        return [self.ctx.device_stats(g) for g in range(len(self.ordinals))]

    def close(self):
        self.ctx.close()
        self.sets = []


def rest(ords, seconds):
    """Let the GPUs idle before a measurement pass. The power limiter reacts to the previous
    pass's load within a fraction of a second: a pass that follows ~0.2 s of full load ran
    every kernel 9-30 % slower (profiles/r02/bench_order/). Each pass then starts in the
    same (burst) state as the timed region."""
    import torch
    for d in set(ords):
        torch.cuda.synchronize(d)
    time.sleep(seconds)


def launches_per_flush(ctx):
    """Kernels launched by the last flush (svp_flush_stats.kernel_launches: every coalesced
    launch op, plus hist256's zeroing kernel and the SGEMM tail split's slice launch and
    reduction when they run)."""
    return int(ctx.flush_stats()["kernel_launches"])


def gpu_plan(args, ws, local):
    """Which CUDA devices this process drives.  torchrun (WORLD_SIZE = N): one GPU per rank.
    Otherwise one process drives all N GPUs through the library's own Job Dispatcher and
    per-GPU workers; SVP_BENCH_DEVICES="0,0" maps N logical GPUs onto given ordinals (a
    1-GPU box can then exercise the N-GPU path; the line says so)."""
    import torch
    N = args.gpus
    if ws > 1:
        if ws != N:
            raise SystemExit(f"--gpus {N} but WORLD_SIZE={ws}: launch one rank per GPU")
        return [local], "process"
    env = os.environ.get("SVP_BENCH_DEVICES")
    if env:
        ords = [int(x) for x in env.split(",") if x.strip()]
        if len(ords) != N:
            raise SystemExit(f"SVP_BENCH_DEVICES lists {len(ords)} devices, --gpus {N}")
    else:
        ords = list(range(N))
    have = torch.cuda.device_count()
    if max(ords) >= have:
        raise SystemExit(f"--gpus {N} needs CUDA devices {ords}, this box has {have}")
    return ords, "single"


def roofline_of(kstats, impl, peaks, peak_src, kchunk=None):
    from paper_conf_dac_jungc15_b200 import svp
    dom = max(kstats, key=lambda n: kstats[n]["total_ns"])
    dk = kstats[dom]
    if dom == "sgemm" and impl == svp.SGEMM_3XTF32:
        bf16 = float(peaks.get("bf16_tflops", 1590.0))
        peak = bf16 * 0.5 / 3.0
        achieved = (dk["flops"] / dk["launches"]) / (dk["total_ns"] / dk["launches"]) / 1e3
        roof = {"kernel": "sgemm 3xTF32 (k_sgemm_tc<3,2>: CTA pairs, tcgen05 kind::tf32)", "bound": "tensor",
                "achieved": achieved, "peak": peak, "unit": "TFLOP/s", "frac": achieved / peak, "traffic": None,
                "peak_source": f"bf16_tflops {bf16:.0f} ({peak_src} burst) x 0.5 (TF32/BF16 nominal) / 3 MMAs per "
                               f"product (3xTF32); achieved counts algorithmic 2MNK flops",
                "tensor_pipe_tflops": 3 * achieved}
    elif dom == "sgemm" and impl == svp.SGEMM_TF32BF16:
        bf16 = float(peaks.get("bf16_tflops", 1590.0))
        peak = bf16 / 4.0
        achieved = (dk["flops"] / dk["launches"]) / (dk["total_ns"] / dk["launches"]) / 1e3
        roof = {"kernel": "sgemm TF32+2xBF16 (k_sgemm_tc<2,2>: CTA pairs, tcgen05 kind::tf32 + kind::f16)",
                "bound": "tensor",
                "achieved": achieved, "peak": peak, "unit": "TFLOP/s", "frac": achieved / peak, "traffic": None,
                "peak_source": f"bf16_tflops {bf16:.0f} ({peak_src} burst) / 4: per product one TF32 MMA (2 BF16 "
                               f"slots at the nominal 1/2 ratio) + two BF16 MMAs; achieved counts 2MNK flops"}
    elif dom == "sgemm":
        sm_mhz = float(peaks.get("sm_max_mhz", 1965.0))
        peak = 148 * 128 * 2 * sm_mhz * 1e6 / 1e12
        achieved = (dk["flops"] / dk["launches"]) / (dk["total_ns"] / dk["launches"]) / 1e3
        roof = {"kernel": "sgemm_ffma (k_sgemm_ffma)", "bound": "alu", "achieved": achieved, "peak": peak,
                "unit": "TFLOP/s", "frac": achieved / peak, "traffic": None,
                "peak_source": f"derived: 148 SM x 128 FP32 lanes x 2 x {sm_mhz:.0f} MHz (sm_max_mhz, {peak_src})"}
    else:
        peak = float(peaks["hbm_gbs"])
        achieved = (dk["bytes"] / dk["launches"]) / (dk["total_ns"] / dk["launches"])
        roof = {"kernel": dom, "bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                "frac": achieved / peak, "traffic": None, "peak_source": f"hbm_gbs ({peak_src})"}
    roof["where"] = ("one-stream pass over the same jobs: each coalesced launch alone on the GPU (the executor "
                     "then runs the SGEMM's partial last wave as the K-split tail and Black-Scholes in dynamic "
                     "tile order); in the interleaved timed step the launches co-run (timed_kernel_ms_per_step)")
    if roof["bound"] == "tensor":
        nominal = 2250.0 * roof["peak"] / float(peaks.get("bf16_tflops", 1590.0))
        roof["peak_nominal"] = nominal
        roof["frac_of_nominal"] = roof["achieved"] / nominal
        if "bf16_tflops_sustained" in peaks:
            sus = float(peaks["bf16_tflops_sustained"]) * roof["peak"] / float(peaks.get("bf16_tflops", 1590.0))
            roof["peak_sustained"] = sus
            roof["frac_of_sustained"] = roof["achieved"] / sus
    # DRAM bytes per launch of the dominant kernel from one committed ncu --set full capture
    # (round 2 first, round-1 figures for kernels not re-captured)
    key = dom + ({svp.SGEMM_3XTF32: "_3xtf32", svp.SGEMM_TF32BF16: "_tf32bf16"}.get(impl, "") if dom == "sgemm" else "")
    if dom == "sgemm" and impl == svp.SGEMM_TF32BF16 and kchunk == 0:
        key += "_kchunk0"
    for name in ("traffic_r02.json", "traffic_r01.json"):
        prof_path = os.path.join(ROOT, "profiles", name)
        try:
            tr = json.load(open(prof_path))
        except Exception:
            continue
        if key in tr:
            roof["traffic"] = tr[key]
            roof["traffic_source"] = f"profiles/{name} (ncu --set full of the cfg5 launch)"
            break
    return dom, roof


def run_svp(args, rank, ws, local):
    import torch
    from paper_conf_dac_jungc15_b200 import svp

    ords, mode = gpu_plan(args, ws, local)
    N = args.gpus
    scaling = args.scaling if args.scaling != "auto" else ("strong" if N > 1 else "weak")
    torch.cuda.set_device(ords[0])
    streams = [torch.cuda.current_stream(d) for d in ords]
    impl = IMPLS[args.sgemm_impl]
    trace(f"mode {mode}, devices {ords}, scaling {scaling}")
    # the workload: BASELINE config k; strong scaling = its VPs split over the N GPUs (the
    # config's definition for cfg5 at 2/4/8 GPUs), weak = N x its VPs
    per_gpu = args.vps or len(W.config_specs(args.config))
    all_specs = W.config_specs(args.config, nvps=per_gpu * (N if scaling == "weak" else 1))
    specs = my_specs(all_specs, rank, ws) if mode == "process" else list(all_specs)
    t_gen = time.perf_counter()
    inputs = W.make_inputs_many(specs)
    t_gen = time.perf_counter() - t_gen
    nsets = n_buffer_sets(all_specs)
    f4 = dict(hetero=bool(args.hetero), graph=bool(args.graph), table_mode=args.table_mode,
              streams_per_gpu=args.streams)

    # ---------------- device-resident run (value)
    # timed at the library's default profile_level 0 (no per-op events); the per-GPU
    # Profiler numbers come from a profiled pass over the same buffers right after
    arm = Arm(specs, inputs, "device", ords, streams, nsets, profile_level=args.timed_profile_level,
              validate_ptrs=True, sgemm_impl=impl, sgemm_kchunk=args.sgemm_kchunk,
              async_flush=bool(args.async_flush), **f4)
    kids = arm.kids
    assert arm.ctx.flush_stats is not None
    arm.step()
    if args.graph:
        # steady state of the plan cache: every buffer set's plan seen twice (planned, then
        # captured), so the timed steps replay graphs (setup, before the W warm-up steps)
        arm.steps(2 * len(arm.batches))
    for d in set(ords):
        torch.cuda.synchronize(d)
    clocks = Clocks(sorted(set(ords)))  # sampling starts before the warm-up (nvidia-smi start-up)
    arm.steps(max(0, args.warmup - 1))
    arm.ctx.reset_profile()
    barrier(ws)
    clocks.mark_start()
    dt, dt_per_gpu = arm.timed(args.steps)
    clocks.mark_end()
    clk = clocks.stop()
    barrier(ws)
    dt_max = max_over_ranks(dt, ws)
    n_jobs_total = sum_over_ranks(len(specs), ws)
    value = n_jobs_total * args.steps / dt_max
    st = arm.ctx.flush_stats()
    launches = launches_per_flush(arm.ctx) * args.steps
    # profiled pass (profile_level 1, same buffers, same options): per-GPU spans, kernel
    # times and the interleaved step's per-kernel times
    if args.timed_profile_level >= 1:
        pa, prof_steps = arm, args.steps
    else:
        pa = Arm(specs, inputs, "device", ords, streams, share=arm, profile_level=1, sgemm_impl=impl,
                 sgemm_kchunk=args.sgemm_kchunk, **f4)
        prof_steps = max(3, min(args.steps, 20))
        rest(ords, args.rest_s)
        pa.steps((2 if args.graph else 1) * len(pa.batches) + 1)
        pa.ctx.reset_profile()
        pa.timed(prof_steps)
    pst = pa.ctx.flush_stats()
    main_kstats = {name: pa.ctx.kernel_stats(kid) for name, kid in kids.items()}
    if args.hetero:
        main_kstats["ew_mix"] = pa.ctx.kernel_stats(svp.KERNEL_EW_MIX)
    dstats = pa.device_stats()
    if pa is not arm:
        pa.close()
    gpus_driven = sum(1 for d in dstats if d["flushes"] > 0)
    per_gpu_rows = []
    for g, (d, t) in enumerate(zip(dstats, dt_per_gpu)):
        per_gpu_rows.append({"gpu": g, "ordinal": d["ordinal"], "vps": d["vps"],
                             "lpt_est_load_ms": d["est_load_ns"] / 1e6,  # VPSet's estimated kernel ns
                             "device_ms_per_step": d["device_ns"] / prof_steps / 1e6,
                             "kernel_ms_per_step": d["kernel_ns"] / prof_steps / 1e6,
                             "event_ms_per_step": t / args.steps * 1e3})
    spans = [r["device_ms_per_step"] for r in per_gpu_rows]
    loads = [r["lpt_est_load_ms"] for r in per_gpu_rows]
    multi = {"mode": mode, "devices": ords, "gpus_driven": gpus_driven if mode == "single" else ws,
             "logical_gpus": len(set(ords)) < len(ords),
             "per_gpu": per_gpu_rows,
             "imbalance_max_over_mean": (max(spans) / (sum(spans) / len(spans))) if spans and sum(spans) else None,
             "lpt_predicted_makespan_ms": max(loads) if loads else None,
             "lpt_predicted_imbalance": (max(loads) / (sum(loads) / len(loads))) if loads and sum(loads) else None}
    if mode == "single":
        assert gpus_driven == N, f"--gpus {N} but the flush ran on {gpus_driven} GPUs"
    trace("timed region done")

    # ---------------- one stream per GPU: per-kernel roofline numbers (launches do not overlap)
    iso = Arm(specs, inputs, "device", ords, streams, share=arm, profile_level=1, interleave=False, sgemm_impl=impl,
              sgemm_kchunk=args.sgemm_kchunk)
    rest(ords, args.rest_s)
    iso.steps(2 * len(iso.batches) + 1)  # (graph replay: every set planned, then captured)
    iso.ctx.reset_profile()
    iso_steps = max(3, args.steps // 5)
    iso_dt, _ = iso.timed(iso_steps)
    kstats = {name: iso.ctx.kernel_stats(kid) for name, kid in iso.kids.items()}
    iso.close()
    iso_value = n_jobs_total * iso_steps / max_over_ranks(iso_dt, ws)
    mb_bytes = sum(k["bytes"] for n, k in kstats.items() if n != "sgemm")
    mb_ns = sum(k["total_ns"] for n, k in kstats.items() if n != "sgemm")
    hbm_gbs = mb_bytes / mb_ns if mb_ns else None
    per_kernel = {}
    tot_k = sum(k["total_ns"] for k in kstats.values())
    for n, k in kstats.items():
        if not k["launches"]:
            continue
        avg = k["total_ns"] / k["launches"]
        row = {"avg_launch_ms": avg / 1e6, "share_of_kernel_time": k["total_ns"] / tot_k if tot_k else None}
        if n == "sgemm":
            row["tflops"] = k["flops"] / k["total_ns"] / 1e3
        else:
            row["gbs"] = k["bytes"] / k["total_ns"]
        per_kernel[n] = row
    peaks, peak_src = measured_peaks()
    dom, roof = roofline_of(kstats, impl, peaks, peak_src, args.sgemm_kchunk)
    if args.config != 5:
        roof["traffic"] = None  # the committed ncu traffic figure is cfg5's launch
        roof.pop("traffic_source", None)

    # ---------------- the other implementations of the fp32 "sgemm" kernel, same jobs (and the
    # selected one with K-chunked accumulation, the strict mode of DESIGN R23)
    alt = []
    if not args.no_alt and "sgemm" in kids:
        variants = [(a, None) for a in args.alt_impl.split(",") if a and IMPLS[a] != impl]
        if args.sgemm_kchunk != 0 and impl != IMPLS["ffma"]:
            variants.append((args.sgemm_impl, 0))  # one accumulation per tile: the cost of R23's chunks
        for alt_name, kc in variants:
            a = Arm(specs, inputs, "device", ords, streams, share=arm, profile_level=1, sgemm_impl=IMPLS[alt_name],
                    sgemm_kchunk=kc)
            rest(ords, args.rest_s)
            a.steps(2 * len(a.batches) + 1)
            a.ctx.reset_profile()
            ks = max(3, args.steps // 5)
            adt = max_over_ranks(a.timed(ks)[0], ws)
            sk = a.ctx.kernel_stats(a.kids["sgemm"])
            alt.append({"sgemm_impl": alt_name, "sgemm_kchunk": kc, "dtype": DTYPE_LABEL[alt_name],
                        "value": n_jobs_total * ks / adt,
                        "unit": "jobs/s", "ms_per_step": adt / ks * 1e3,
                        "sgemm_tflops_interleaved": (sk["flops"] / sk["total_ns"] / 1e3) if sk["total_ns"] else None})
            a.close()
    trace("alt pass done")

    # ---------------- serial baselines on the same GPUs, same buffers, same kernels
    serial, by_kernel = {}, {}
    if not args.no_serial:
        for name, kw in (("B1_serial_sync", dict(coalesce=False, interleave=False, sync_each_job=True, graph=False)),
                         ("B2_serial_async", dict(coalesce=False, interleave=False, graph=False)),
                         ("B3_serial_graph", dict(coalesce=False, interleave=False, graph=True)),
                         ("B2_profiled", dict(coalesce=False, interleave=False, profile_level=1, graph=False))):
            # same buffer sets as the coalesced arm; B3 replays one captured graph per set
            b = Arm(specs, inputs, "device", ords, streams, share=arm, sgemm_impl=impl,
                    sgemm_kchunk=args.sgemm_kchunk, **kw)
            # B3: each set's plan, then its capture + instantiate, then replays only
            rest(ords, args.rest_s)
            b.steps(max(3, args.warmup) + (2 * len(b.batches) if kw.get("graph") else 0))
            b.ctx.reset_profile()
            barrier(ws)
            ks = max(2, args.steps // 5)
            sdt = max_over_ranks(b.timed(ks)[0], ws)
            if name != "B2_profiled":
                serial[name] = {"value": n_jobs_total * ks / sdt, "unit": "jobs/s", "steps": ks,
                                "ms_per_step": sdt / ks * 1e3}
            else:
                # Eq 9's alignment gain per kernel class: per-job launches vs one coalesced
                # launch of the same jobs (event-timed kernel time per step, 1 stream each)
                for kname, kid in b.kids.items():
                    st_ser = b.ctx.kernel_stats(kid)
                    st_coal = kstats[kname]
                    if st_ser["launches"] and st_coal["launches"]:
                        ser_ms = st_ser["total_ns"] / ks / 1e6
                        coal_ms = st_coal["total_ns"] / iso_steps / 1e6
                        by_kernel[kname] = {"serial_kernel_ms": ser_ms, "coalesced_kernel_ms": coal_ms,
                                            "speedup": ser_ms / coal_ms}
            b.close()
    arm.close()
    torch.cuda.empty_cache()
    trace("serial passes done")

    # ---------------- e2e: pinned host buffers, copies inside the timed region
    e2e = None
    if not args.no_e2e:
        h = Arm(specs, inputs, "host", ords, streams, 1, arena_bytes=args.arena_gb << 30, sgemm_impl=impl,
                sgemm_kchunk=args.sgemm_kchunk, host_numa=bool(args.host_numa), async_flush=bool(args.async_flush),
                max_chunks=int(os.environ.get("SVP_BENCH_MAXCH", "8")), **f4)
        h.steps(2)
        hst = h.ctx.flush_stats()
        barrier(ws)
        ks = args.e2e_steps or max(2, min(args.steps, 5))
        edt = max_over_ranks(h.timed(ks)[0], ws)
        e2e = {"value": n_jobs_total * ks / edt, "unit": "jobs/s",
               "h2d_bytes_per_step": int(sum_over_ranks(hst["h2d_bytes"], ws)),
               "d2h_bytes_per_step": int(sum_over_ranks(hst["d2h_bytes"], ws)),
               "steps": ks, "ms_per_step": edt / ks * 1e3, "chunks": int(hst["chunks"]),
               "api": "svp_submit_batch + svp_flush, HOST_PINNED buffers (H2D/D2H staged + interleaved)",
               "host_buffers": ("svp_host_alloc on each VP's GPU's NUMA node (node %s)"
                                % sorted({h.ctx.device_stats(g)["numa_node"] for g in range(len(ords))})
                                if args.host_numa else "torch pinned (cudaHostAlloc, first-touch placement)")}
        h.close()

    # ---------------- weak scaling beside the strong number (N > 1)
    weak = None
    if N > 1 and scaling == "strong" and not args.no_weak:
        wspecs_all = W.config_specs(args.config, nvps=per_gpu * N)
        wspecs = my_specs(wspecs_all, rank, ws) if mode == "process" else wspecs_all
        winputs = W.make_inputs_many(wspecs)
        w = Arm(wspecs, winputs, "device", ords, streams, n_buffer_sets(wspecs_all), sgemm_impl=impl,
                sgemm_kchunk=args.sgemm_kchunk, **f4)
        w.steps(args.warmup)
        barrier(ws)
        ks = max(3, args.steps // 3)
        wdt = max_over_ranks(w.timed(ks)[0], ws)
        weak = {"value": sum_over_ranks(len(wspecs), ws) * ks / wdt, "unit": "jobs/s", "vps": len(wspecs_all),
                "steps": ks, "ms_per_step": wdt / ks * 1e3, "scaling": "weak"}
        w.close()
        del winputs

    cpu = None
    if rank == 0 and N == 1 and not args.no_cpu:
        cpu = cpu_baseline(specs, inputs, CONFIG_NAMES[args.config])

    total_launches = int(sum_over_ranks(launches, ws))  # collective: every rank calls it
    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "jobs/s", "n_gpus": N, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": dt_max / args.steps * 1e3, "higher_is_better": True,
            "scaling": scaling, "vs_baseline": None, "dtype": DTYPE_LABEL[args.sgemm_impl],
            "data": "synthetic",
            "config": {"workload": CONFIG_NAMES[args.config], "config_index": args.config, "vps": len(all_specs),
                       "residency": "device (HBM)",
                       "parallelism": (f"dp{N}: VPs sharded by the Job Dispatcher's kernel-stratified LPT, "
                                       + ("one process driving all GPUs (per-GPU worker threads)" if mode == "single"
                                          else "one rank per GPU")),
                       "l2": l2_note(all_specs, nsets)},
            "clocks": clk, "e2e": e2e, "gpu_launches": total_launches,
            "roofline": roof, "cpu_baseline": cpu,
            "multi_gpu": multi, "weak_scaling": weak,
            "hbm_gbs_membound": hbm_gbs,
            "hbm_frac_membound": (hbm_gbs / float(peaks["hbm_gbs"])) if hbm_gbs else None,
            "elements_per_s": sum(s.n for s in all_specs) * args.steps / dt_max,
            "sgemm_impl": args.sgemm_impl, "sgemm_kchunk": args.sgemm_kchunk, "alt_sgemm_impls": alt, "hetero": args.hetero, "graph": args.graph,
            "async_flush": args.async_flush,
            "table_mode": args.table_mode,
            "graph_replays_last_step": int(st["graph_replays"]),
            "timed_kernel_ms_per_step": {n: k["total_ns"] / prof_steps / 1e6 for n, k in main_kstats.items()
                                         if k["launches"]},
            "speedup_vs_serial": {k: value / v["value"] for k, v in serial.items()},
            "serial": serial, "speedup_by_kernel_class": by_kernel, "per_kernel": per_kernel,
            "one_stream": {"value": iso_value, "unit": "jobs/s",
                           "note": "coalesced, 1 compute stream (no interleaving); per_kernel/roofline timed here"},
            "flush": {"host_plan_us": st["host_plan_ns"] / 1e3, "host_issue_us": st["host_issue_ns"] / 1e3,
                      "host_total_us": st["host_total_ns"] / 1e3, "device_ms": pst["device_ns"] / 1e6,
                      "timed_profile_level": args.timed_profile_level,
                      "groups": int(st["groups"]), "launch_ops": int(st["launches"])},
            "parity": "tests/test_gpu_parity.py, test_gpu_sgemm_*.py (full-size configs vs oracle; not re-run here)",
            "profiler_split": "per-VP attribution inside a coalesced launch: parity unpinned (DESIGN.md §3)",
            "setup_s": {"input_generation": t_gen},
        }
        print(json.dumps(line), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=30)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="svp", choices=["svp", "reference"])
    ap.add_argument("--config", type=int, default=5)
    ap.add_argument("--vps", type=int, default=None)
    ap.add_argument("--e2e-steps", type=int, default=0)
    ap.add_argument("--arena-gb", type=int, default=8)
    ap.add_argument("--sgemm-impl", default="tf32bf16", choices=list(IMPL_NAMES),
                    help="implementation of the fp32 'sgemm' kernel (all meet its 1e-5 contract)")
    ap.add_argument("--sgemm-kchunk", type=int, default=None,
                    help="svp_config.sgemm_kchunk: K chunk of the tensor-core accumulation (DESIGN R23); "
                         "default: the library's (768); 0 = one accumulation per tile")
    ap.add_argument("--alt-impl", default="3xtf32,ffma",
                    help="comma list of the other sgemm implementations timed beside the main one")
    ap.add_argument("--scaling", default="auto", choices=["auto", "weak", "strong"],
                    help="auto: strong at N > 1 (the config's VPs split over N GPUs, as BASELINE cfg5 states), "
                         "weak at N = 1; weak: N x the config's VPs (fixed work per GPU)")
    ap.add_argument("--no-weak", action="store_true", help="N > 1: skip the extra weak-scaling measurement")
    ap.add_argument("--hetero", type=int, default=0, choices=[0, 1],
                    help="heterogeneous coalescing of vecadd/SAXPY/Black-Scholes (NEXT f4)")
    ap.add_argument("--graph", type=int, default=1, choices=[0, 1],
                    help="plan cache + CUDA graph replay (NEXT f4; the library default since ABI 6)")
    ap.add_argument("--table-mode", type=int, default=1, choices=[0, 1],
                    help="segment tables: 0 global device buffer, 1 by-value kernel parameter")
    ap.add_argument("--host-numa", type=int, default=1, choices=[0, 1],
                    help="e2e: host buffers from svp_host_alloc on the VP's GPU's NUMA node (0: torch pinned)")
    ap.add_argument("--timed-profile-level", type=int, default=0, choices=[0, 1, 2],
                    help="profile_level of the timed context (default 0, the library default: no per-op events; "
                         "per-GPU / per-kernel numbers then come from a profiled pass over the same buffers)")
    ap.add_argument("--rest-s", type=float, default=1.0,
                    help="idle seconds before each measurement pass after the timed region (power-limiter reset)")
    ap.add_argument("--async-flush", type=int, default=1, choices=[0, 1],
                    help="timed and e2e loops use svp_flush_async (step i's device work overlaps step i+1's host work)")
    ap.add_argument("--streams", type=int, default=4, help="compute streams per GPU (svp_config.streams_per_gpu)")
    ap.add_argument("--no-serial", action="store_true")
    ap.add_argument("--no-alt", action="store_true", help="skip timing the other sgemm implementation")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    args = ap.parse_args()
    if args.warmup < 3:
        print("warning: --warmup < 3 violates the timing rules; using 3", file=sys.stderr)
        args.warmup = 3
    if args.impl == "reference":
        # rank 0 alone runs the oracle arm; other ranks exit without work or rendezvous
        rank, ws = int(os.environ.get("RANK", "0")), int(os.environ.get("WORLD_SIZE", "1"))
        run_reference(args, rank, ws)
        return
    rank, ws, local = dist_setup()
    run_svp(args, rank, ws, local)
    if ws > 1:
        import torch.distributed as dist
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
