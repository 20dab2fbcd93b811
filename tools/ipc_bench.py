"""S7: the IPC front end under load (NEXT f3; PAPER.md L231-235 IPC manager, L240-241
continuous queue).  P VP processes (no CUDA in them), each driving V VPs, issue rounds of
synchronous SAXPY calls on buffers in the shared arena (host-resident: every call is
H2D + kernel + D2H); the server's continuous dispatcher coalesces whatever the processes
have queued.  Reported per P: jobs/s over all processes, mean time of one round (V calls
submitted, then all waited), kernel launches per job (coalescing across processes), and
the same program from V*P in-process VP threads (svp_submit + svp_wait, f1) as reference.

    python tools/ipc_bench.py [--out F] [--n 65536] [--calls 50]
"""
import argparse
import json
import multiprocessing as mp
import os
import sys
import threading
import time
import uuid

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def _vp_process(name, vps, calls, n, q, go):
    try:
        import ctypes

        import numpy as np
        from paper_conf_dac_jungc15_b200 import svp
        c = svp.IpcClient(name)
        k = svp.kernel_lookup("saxpy")
        bufs, ys = [], []
        for v in vps:
            (ox, px), (oy, py) = c.alloc(4 * n), c.alloc(4 * n)
            np.ctypeslib.as_array((ctypes.c_float * n).from_address(px))[:] = 1.0
            y = np.ctypeslib.as_array((ctypes.c_float * n).from_address(py))
            y[:] = 0.0
            ys.append(y)
            bufs.append([(ox, 4 * n, svp.DIR_IN), (oy, 4 * n, svp.DIR_INOUT)])
        args = [svp.args_saxpy(n, 1.0) for _ in vps]
        q.put(("ready", None))
        go.wait()
        t0 = time.perf_counter()
        for _ in range(calls):
            ts = [c.submit(v, k, args[i], bufs[i]) for i, v in enumerate(vps)]
            for t in ts:
                c.wait(t, timeout_ms=120000)
        dt = time.perf_counter() - t0
        ok = all(bool(np.all(y == float(calls))) for y in ys)  # y = calls * 1.0 * 1.0, exact
        c.close()
        q.put(("done", (dt, ok)))
    except Exception as e:  # pragma: no cover
        q.put(("err", repr(e)))


def run_ipc(P, V, calls, n, dry=False):
    from paper_conf_dac_jungc15_b200 import svp
    name = "svp_bench_" + uuid.uuid4().hex[:10]
    ctx = svp.Context(num_gpus=1, profile_level=1, dry_run=dry)
    ctx.register_kernel("saxpy")
    with svp.IpcServer(ctx, name, arena_bytes=max(64 << 20, 2 * P * V * 4 * n + (16 << 20)), nslots=1024) as srv:
        mpx = mp.get_context("spawn")
        q = mpx.Queue()
        go = mpx.Event()
        procs = [mpx.Process(target=_vp_process, args=(name, list(range(V * p, V * p + V)), calls, n, q, go))
                 for p in range(P)]
        for p in procs:
            p.start()
        for _ in procs:
            tag, val = q.get(timeout=300)
            assert tag == "ready", val
        ctx.reset_profile()
        t0 = time.perf_counter()
        go.set()
        res = [q.get(timeout=600) for _ in procs]
        wall = time.perf_counter() - t0
        for p in procs:
            p.join(60)
        assert all(r[0] == "done" for r in res), res
        served = srv.stats()["served"]
    prof = ctx.profile(-1)
    ctx.close()
    jobs = P * V * calls
    return {"procs": P, "vps_per_proc": V, "calls": calls, "n": n, "jobs": jobs, "served": served,
            "wall_s": wall, "jobs_per_s": jobs / wall,
            "round_ms_mean": 1e3 * sum(r[1][0] for r in res) / len(res) / calls,
            "results_ok": all(r[1][1] for r in res),
            "launches": prof["launches"], "launches_per_job": prof["launches"] / max(1, prof["jobs"])}


def run_threads(T, calls, n):
    """The same program from T in-process VP threads (f1: svp_submit + svp_wait with the
    continuous dispatcher), host-pinned buffers."""
    import torch
    from paper_conf_dac_jungc15_b200 import svp
    ctx = svp.Context(num_gpus=1, profile_level=1)
    k = ctx.register_kernel("saxpy")
    xs = [torch.ones(n, pin_memory=True) for _ in range(T)]
    ys = [torch.zeros(n, pin_memory=True) for _ in range(T)]
    ctx.start_dispatcher()
    ctx.reset_profile()
    bar = threading.Barrier(T + 1)

    def vp(i):
        bar.wait()
        for _ in range(calls):
            j = ctx.submit(i, k, svp.args_saxpy(n, 1.0), [(xs[i].data_ptr(), 4 * n, svp.DIR_IN, svp.MEM_HOST_PINNED),
                                                          (ys[i].data_ptr(), 4 * n, svp.DIR_INOUT,
                                                           svp.MEM_HOST_PINNED)])
            ctx.wait(j, 120000)

    th = [threading.Thread(target=vp, args=(i,)) for i in range(T)]
    for t in th:
        t.start()
    bar.wait()
    t0 = time.perf_counter()
    for t in th:
        t.join()
    wall = time.perf_counter() - t0
    ctx.stop_dispatcher()
    prof = ctx.profile(-1)
    ok = all(bool((y == float(calls)).all()) for y in ys)
    ctx.close()
    jobs = T * calls
    return {"threads": T, "calls": calls, "n": n, "jobs": jobs, "wall_s": wall, "jobs_per_s": jobs / wall,
            "results_ok": ok, "launches_per_job": prof["launches"] / max(1, prof["jobs"])}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=None)
    ap.add_argument("--n", type=int, default=1 << 16)
    ap.add_argument("--calls", type=int, default=50)
    ap.add_argument("--vps", type=int, default=4)
    ap.add_argument("--dry", action="store_true", help="dry-run server (host logic only, no results)")
    args = ap.parse_args()
    out = {"ipc": [], "threads": []}
    for P in (1, 2, 4, 8):
        r = run_ipc(P, args.vps, args.calls, args.n, args.dry)
        print(json.dumps(r), flush=True)
        out["ipc"].append(r)
        if args.dry:
            continue
        t = run_threads(P * args.vps, args.calls, args.n)
        print(json.dumps(t), flush=True)
        out["threads"].append(t)
    if args.out:
        json.dump(out, open(args.out, "w"), indent=1)


if __name__ == "__main__":
    main()
