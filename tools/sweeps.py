"""Reproduce the paper's coalescing / interleaving experiments on B200 with libsvp.

    python tools/sweeps.py [--out profiles/r01/sweeps.json] [--quick]

S1 (Fig 10a): vectorAdd, constant total 2^26 elements split over N
    VPs; one coalesced flush vs the same N jobs launched serially (B1: one launch per job,
    sync after each; B2: no syncs).  Paper (Quadro 4000): 10.54x at N=16, 20.48x at N=64.
S2 (Fig 10b + Eq 9): one vecadd VP of n = k tiles; kernel time vs k
    is a staircase with step lambda = #SMs x resident CTAs (Eq 9's aligned unit).
S3 (Fig 9 + Eq 7/8): N host-resident SGEMM jobs (H2D A,B -> kernel ->
    D2H C) with Tk ~ Tm, interleaved on separate copy/compute streams vs one stream;
    measured speedup next to Eq 7's prediction from the measured Tm, Tk.
S3a (Fig 9a): two interleaved host-resident programs, input size fixed,
    kernel length varied (tensor-core SGEMM K-chunk count, FFMA); speedup vs Tk / Tm.  Run
    with --only a (not in the default set).
S4 (BASELINE metric): jobs/s of the cfg5 mix vs #VPs (1 GPU).
S5 (Table 1): N VPs each running the paper's program -- 300
    multiplications of two 320x320 fp64 matrices -- coalesced per program-order level vs
    serial per-VP launches; DGEMM TFLOP/s; the same program with steady-state graph replay.
S6 (NEXT f4, launch-bound mixes): N VPs with small vecadd / SAXPY / Black-Scholes jobs
    (16Ki-64Ki elements); wall time of submit + flush per round for the default path,
    hetero (one mixed launch), graph (plan reuse + CUDA-graph replay), graph with pipelined
    flushes (svp_flush_async, rounds back to back), both, and the serial baselines B2 / B3
    (B2 as a graph).
Times are CUDA-event device times around whole flushes (median of reps).
"""
import argparse
import json
import os
import statistics
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import workloads as W  # noqa: E402
from paper_conf_dac_jungc15_b200 import svp  # noqa: E402
from paper_conf_dac_jungc15_b200.vpset import VPSet  # noqa: E402


def flush_time(ctx, jobs, reps=5, warm=2):
    s = torch.cuda.current_stream()
    jobs = svp.JobBatch(jobs)
    for _ in range(warm):
        ctx.submit_batch(jobs)
        ctx.flush()
    ts = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record(s)
        ctx.submit_batch(jobs)
        ctx.flush()
        e1.record(s)
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) / 1e3)
    return statistics.median(ts)


def ctx_for(**kw):
    # SVP_SWEEP_VALIDATE: validate_ptrs level of every context (A/B of the range cache)
    kw.setdefault("validate_ptrs", int(os.environ.get("SVP_SWEEP_VALIDATE", "1")))
    kw.setdefault("graph", False)  # the paper's experiments: plain flushes unless a row asks for replay
    return svp.Context(num_gpus=1, external_streams=[torch.cuda.current_stream().cuda_stream], **kw)


def s1_coalescing(quick):
    total = 1 << 26
    out = []
    for N in ([1, 4, 16, 64] if quick else [1, 2, 4, 8, 16, 32, 64, 128, 256]):
        specs = [W.JobSpec(v, "vecadd", n=total // N) for v in range(N)]
        c = ctx_for()
        vs = VPSet(c, specs, [W.make_inputs(s) for s in specs], "device")
        jobs = vs.job_list()
        t_coal = flush_time(c, jobs)
        row = {"N": N, "coalesced_ms": t_coal * 1e3}
        for name, kw in (("B1_serial_sync", dict(coalesce=False, interleave=False, sync_each_job=True)),
                         ("B2_serial_async", dict(coalesce=False, interleave=False))):
            sc = ctx_for(**kw)
            sc.register_kernel("vecadd")
            t = flush_time(sc, jobs)
            row[name + "_ms"] = t * 1e3
            row["speedup_vs_" + name] = t / t_coal
            sc.close()
        row["coalesced_gbs"] = 12 * total / t_coal / 1e9
        out.append(row)
        c.close()
        del vs
        torch.cuda.empty_cache()
    return out


def s2_staircase(quick):
    c = ctx_for(profile_level=1, interleave=False)
    kid = c.register_kernel("vecadd")
    lim_tile = 4096
    props = torch.cuda.get_device_properties(0)
    rows = []
    ks = list(range(148, 148 * 8 * 3 + 1, 148 if quick else 74))
    nmax = max(ks) * lim_tile
    a = torch.rand(nmax, device="cuda")
    b = torch.rand(nmax, device="cuda")
    cc = torch.empty(nmax, device="cuda")
    for k in ks:
        n = k * lim_tile
        job = (0, kid, svp.args_vecadd(n), [(a.data_ptr(), 4 * n, 1, 0), (b.data_ptr(), 4 * n, 1, 0),
                                            (cc.data_ptr(), 4 * n, 2, 0)])
        c.reset_profile()
        flush_time(c, [job], reps=7)
        st = c.kernel_stats(kid)
        rows.append({"tiles": k, "elements": n, "kernel_us": st["total_ns"] / st["launches"] / 1e3})
    c.close()
    return {"sms": props.multi_processor_count, "tile_elements": lim_tile, "rows": rows}


def s3_interleaving(quick):
    """N host-resident FFMA SGEMMs of n^3 with Tk ~ Tm (Fig 9b); no coalescing, so only the
    Copy/Compute-engine interleaving differs between the two runs."""
    n = 3072
    rows = []
    for N in ([2, 4, 8] if quick else [2, 4, 8, 16, 32]):
        specs = [W.JobSpec(v, "sgemm", M=n, N=n, K=n) for v in range(N)]
        inputs = [W.make_inputs(s) for s in specs]
        res = {}
        for name, kw in (("interleaved", dict(coalesce=False, interleave=True)),
                         ("serial", dict(coalesce=False, interleave=False))):
            c = ctx_for(sgemm_impl=svp.SGEMM_FFMA, profile_level=1, arena_bytes=8 << 30, **kw)
            vs = VPSet(c, specs, inputs, "host")
            t = flush_time(c, vs.job_list(), reps=3, warm=1)
            res[name] = t
            if name == "serial":
                ops = c.plan()
                tin = statistics.median([o["measured_ns"] for o in ops if o["kind"] == svp.OP_H2D]) / 1e6
                tk = statistics.median([o["measured_ns"] for o in ops if o["kind"] == svp.OP_KERNEL]) / 1e6
                tout = statistics.median([o["measured_ns"] for o in ops if o["kind"] == svp.OP_D2H]) / 1e6
            c.close()
            del vs
            torch.cuda.empty_cache()
        tm = tin
        eq7 = 2 * tm + N * max(tm, tk)
        rows.append({"N": N, "Tin_ms": tin, "Tk_ms": tk, "Tout_ms": tout, "serial_ms": res["serial"] * 1e3,
                     "interleaved_ms": res["interleaved"] * 1e3, "speedup": res["serial"] / res["interleaved"],
                     "eq7_pred_ms": eq7, "eq8_speedup_if_equal": 3 * N / (2 + N)})
    return {"sgemm_n": n, "rows": rows}


def s3a_kernel_length(quick):
    """Fig 9(a): two interleaved programs (H2D -> kernel -> D2H), the input
    size fixed and the kernel's length varied.  Every point is the same 3072^3 host-resident
    SGEMM per program (so Tm is the same), and the kernel length is set by the tensor-core
    SGEMM's K-chunk count (sgemm_kchunk: each chunk's partial sums are folded into C, so
    more chunks = a longer kernel computing the same product), the FFMA kernel and the
    plain-load kernel.  Serial vs interleaved with the measured Tm, Tk; Eq 7's prediction
    2 Tm + N max(Tm, Tk), and the three-engine flow-shop bound."""
    n, N = 3072, 2
    variants = [("tf32bf16", svp.SGEMM_TF32BF16, kc, n) for kc in
                ([1536, 256, 64, 16] if quick else [1536, 1024, 512, 256, 128, 64, 32, 16])]
    variants.append(("ffma", svp.SGEMM_FFMA, None, n))
    # K = n - 1: a row pitch TMA cannot address -> the plain-load kernel (shape key 2), the
    # slowest of the four; its copies are 1/n (0.03 %) shorter than the others'
    variants.append(("plain_load", svp.SGEMM_FFMA, None, n - 1))
    rows = []
    for label, impl, kc, K in variants:
        specs = [W.JobSpec(v, "sgemm", M=n, N=n, K=K) for v in range(N)]
        inputs = [W.make_inputs(s) for s in specs]
        res = {}
        for name, kw in (("interleaved", dict(coalesce=False, interleave=True)),
                         ("serial", dict(coalesce=False, interleave=False))):
            c = ctx_for(sgemm_impl=impl, sgemm_kchunk=kc, profile_level=1, arena_bytes=4 << 30, **kw)
            vs = VPSet(c, specs, inputs, "host")
            res[name] = flush_time(c, vs.job_list(), reps=3, warm=1)
            if name == "serial":
                ops = c.plan()
                tin = statistics.median([o["measured_ns"] for o in ops if o["kind"] == svp.OP_H2D]) / 1e6
                tk = statistics.median([o["measured_ns"] for o in ops if o["kind"] == svp.OP_KERNEL]) / 1e6
                tout = statistics.median([o["measured_ns"] for o in ops if o["kind"] == svp.OP_D2H]) / 1e6
            c.close()
            del vs
            torch.cuda.empty_cache()
        rows.append({"kernel": label, "sgemm_kchunk": kc, "K": K, "Tin_ms": tin, "Tk_ms": tk, "Tout_ms": tout,
                     "Tk_over_Tm": tk / tin, "serial_ms": res["serial"] * 1e3,
                     "interleaved_ms": res["interleaved"] * 1e3, "speedup": res["serial"] / res["interleaved"],
                     "eq7_pred_ms": 2 * tin + N * max(tin, tk),
                     "eq7_pred_speedup": res["serial"] * 1e3 / (2 * tin + N * max(tin, tk)),
                     # three engines (H2D copy, compute, D2H copy) as a flow shop of N identical
                     # programs: the first program's three stages + (N - 1) x the slowest stage
                     "flowshop_pred_ms": tin + tk + tout + (N - 1) * max(tin, tk, tout)})
    rows.sort(key=lambda r: r["Tk_ms"])
    return {"sgemm_n": n, "programs": N, "rows": rows}


def s4_vps(quick):
    """BJ metric vs #VPs at G = 1: jobs/s of the cfg5 prefix with nv VPs (all kernels), and
    HBM GB/s of its memory-bound VPs flushed on their own (algorithmic bytes / device span
    of the flush, profile_level 1 events)."""
    rows = []
    for nv in ([16, 64, 256] if quick else [2, 4, 8, 16, 32, 64, 128, 256]):
        specs = W.config_specs(5, nvps=nv)
        c = ctx_for()
        vs = VPSet(c, specs, W.make_inputs_many(specs), "device")
        t = flush_time(c, vs.job_list(), reps=5)
        row = {"vps": nv, "ms": t * 1e3, "jobs_per_s": nv / t}
        c.close()
        del vs
        mem = [s for s in specs if s.kernel in W.MEMBOUND]
        if mem:
            c = ctx_for(profile_level=1)
            vs = VPSet(c, mem, W.make_inputs_many(mem), "device")
            jobs = vs.job_list()
            flush_time(c, jobs, reps=3)
            dev = []
            for _ in range(5):
                c.submit_batch(svp.JobBatch(jobs))
                c.flush()
                dev.append(c.flush_stats()["device_ns"])
            # algorithmic bytes: 12 B/elem vecadd, SAXPY; 20 B/option BS;
            # 1 B/byte + the 1-KiB counts for hist256
            nbytes = sum(12 * s.n if s.kernel in ("vecadd", "saxpy") else 20 * s.n if s.kernel == "blackscholes"
                         else s.n + (1024 if s.n else 0) for s in mem)
            row["membound_vps"] = len(mem)
            row["membound_device_ms"] = statistics.median(dev) / 1e6
            row["membound_hbm_gbs"] = nbytes / (statistics.median(dev) * 1e-9) / 1e9
            c.close()
            del vs
        rows.append(row)
        torch.cuda.empty_cache()
    return rows


def s5_table1(quick):
    iters = 100 if quick else 300
    rows = []
    for nv in ([1, 8] if quick else [1, 2, 4, 8, 16, 32]):
        specs = W.table1_specs(nvps=nv, iters=iters)
        base = [W.make_inputs(s) for s in specs[::iters]]
        c = ctx_for(profile_level=1)
        # every job of a VP reuses the VP's A, B, C buffers (the program's loop body)
        vs = VPSet(c, specs[::iters], base, "device")
        one = vs.job_list()
        jobs = [one[i // iters] for i in range(len(specs))]
        c.reset_profile()
        t = flush_time(c, jobs, reps=3, warm=1)
        ks = c.kernel_stats(c.kernel_ids["dgemm"])
        row = {"vps": nv, "iters": iters, "coalesced_ms": t * 1e3, "jobs_per_s": len(jobs) / t,
               "dgemm_tflops_kernel": ks["flops"] / ks["total_ns"] / 1e3 if ks["total_ns"] else None,
               "launches_per_flush": c.flush_stats()["launches"]}
        sc = ctx_for(coalesce=False, interleave=False, sync_each_job=True)
        sc.register_kernel("dgemm")
        ts = flush_time(sc, jobs, reps=1, warm=1)
        sc.close()
        gc = ctx_for(graph=True)
        gc.register_kernel("dgemm")
        row["graph_ms"] = flush_time(gc, jobs, reps=3, warm=2) * 1e3
        row["graph_wall_ms"] = wall_time(gc, jobs, reps=3, warm=1) * 1e3
        row["coalesced_wall_ms"] = wall_time(c, jobs, reps=3, warm=1) * 1e3
        gc.close()
        row["serial_sync_ms"] = ts * 1e3
        row["speedup_vs_serial_sync"] = ts / t
        rows.append(row)
        c.close()
        del vs
        torch.cuda.empty_cache()
    return {"paper_table1_ms": {"native_gpu_quadro4000": 170.79, "sigma_vp": 568.12, "emul_on_cpu": 9141.51},
            "rows": rows}


def wall_time(ctx, jobs, reps=50, warm=5):
    """Host wall time of submit + flush (the flush returns when the outputs are in place)."""
    import time
    jobs = svp.JobBatch(jobs)
    for _ in range(warm):
        ctx.submit_batch(jobs)
        ctx.flush()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        t0 = time.perf_counter()
        ctx.submit_batch(jobs)
        ctx.flush()
        ts.append(time.perf_counter() - t0)
    return statistics.median(ts)


def pipelined_time(ctx, jobs, reps=200, warm=10):
    """Host wall time per round of submit + svp_flush_async, rounds back to back (each
    round's device work overlaps the next round's host work); the last is waited for."""
    import time
    jobs = svp.JobBatch(jobs)
    for _ in range(warm):
        ctx.submit_batch(jobs)
        t = ctx.flush_async()
    ctx.flush_wait(t)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(reps):
        ctx.submit_batch(jobs)
        t = ctx.flush_async()
    ctx.flush_wait(t)
    return (time.perf_counter() - t0) / reps


def s6_f4(quick):
    kinds = ("vecadd", "saxpy", "blackscholes")
    rows = []
    for nv in ([16, 256] if quick else [16, 64, 256, 1024]):
        g = np.random.default_rng(nv)
        specs = [W.JobSpec(v, kinds[v % 3], n=int(g.integers(1 << 14, 1 << 16)), R=0.02, V=0.3,
                           a=float(g.uniform(-2, 2))) for v in range(nv)]
        inputs = W.make_inputs_many(specs)
        row = {"vps": nv, "elements": int(sum(s.n for s in specs))}
        for name, kw in (("default", {}), ("hetero", dict(hetero=True)), ("graph", dict(graph=True)),
                         ("hetero_graph", dict(hetero=True, graph=True)),
                         ("B2_serial_async", dict(coalesce=False, interleave=False)),
                         ("B3_serial_graph", dict(coalesce=False, interleave=False, graph=True))):
            c = ctx_for(**kw)
            vs = VPSet(c, specs, inputs, "device")
            t = wall_time(c, vs.job_list())
            st = c.flush_stats()
            if name == "graph":  # the same rounds pipelined (svp_flush_async)
                row["graph_async_us"] = pipelined_time(c, vs.job_list()) * 1e6
            row[name + "_us"] = t * 1e6
            row[name + "_launches"] = int(st["launches"])
            row[name + "_host_plan_us"] = st["host_plan_ns"] / 1e3
            row[name + "_host_issue_us"] = st["host_issue_ns"] / 1e3
            c.close()
            del vs
        row["speedup_graph_vs_default"] = row["default_us"] / row["graph_us"]
        row["speedup_graph_async_vs_default"] = row["default_us"] / row["graph_async_us"]
        row["speedup_graph_async_vs_B2"] = row["B2_serial_async_us"] / row["graph_async_us"]
        row["speedup_hetero_graph_vs_default"] = row["default_us"] / row["hetero_graph_us"]
        row["speedup_default_vs_B2"] = row["B2_serial_async_us"] / row["default_us"]
        rows.append(row)
        torch.cuda.empty_cache()
    return rows


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=None)
    ap.add_argument("--quick", action="store_true")
    ap.add_argument("--only", default="123456")
    args = ap.parse_args()
    torch.cuda.set_device(0)
    res = {"gpu": torch.cuda.get_device_name(0)}
    if "1" in args.only:
        res["S1_coalescing_fig10a"] = s1_coalescing(args.quick)
    if "2" in args.only:
        res["S2_staircase_fig10b"] = s2_staircase(args.quick)
    if "3" in args.only:
        res["S3_interleaving_fig9"] = s3_interleaving(args.quick)
    if "a" in args.only:
        res["S3a_kernel_length_fig9a"] = s3a_kernel_length(args.quick)
    if "4" in args.only:
        res["S4_jobs_vs_vps"] = s4_vps(args.quick)
    if "5" in args.only:
        res["S5_table1_dgemm"] = s5_table1(args.quick)
    if "6" in args.only:
        res["S6_f4_launch_bound"] = s6_f4(args.quick)
    txt = json.dumps(res, indent=1)
    print(txt)
    if args.out:
        with open(args.out, "w") as f:
            f.write(txt + "\n")


if __name__ == "__main__":
    main()
