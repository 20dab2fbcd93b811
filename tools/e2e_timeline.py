"""Measured timeline of one host-resident (mode H) flush: where the end-to-end time goes.

    python tools/e2e_timeline.py [--config 5] [--max-chunks 8] [--out FILE]

Runs the config with HOST_PINNED buffers (profile_level 1), repeats the flush a few times
and prints, for the last one, every op's event-timed start / duration on its stream, the
busy time of the H2D and D2H copy streams, the time both directions overlap, the achieved
GB/s per direction, the gaps on the H2D stream, and the flush span against the PCIe floor
(H2D bytes / measured one-direction rate).
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import workloads as W  # noqa: E402
from paper_conf_dac_jungc15_b200 import svp  # noqa: E402
from paper_conf_dac_jungc15_b200.vpset import VPSet  # noqa: E402


def union_len(iv):
    iv = sorted(iv)
    tot, cur_s, cur_e = 0.0, None, None
    for s, e in iv:
        if cur_e is None or s > cur_e:
            if cur_e is not None:
                tot += cur_e - cur_s
            cur_s, cur_e = s, e
        else:
            cur_e = max(cur_e, e)
    if cur_e is not None:
        tot += cur_e - cur_s
    return tot


def intersect_len(a, b):
    tot = 0.0
    for s1, e1 in a:
        for s2, e2 in b:
            tot += max(0.0, min(e1, e2) - max(s1, s2))
    return tot


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=5)
    ap.add_argument("--max-chunks", type=int, default=8)
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--streams", type=int, default=4)
    ap.add_argument("--profile", type=int, default=1)
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    torch.cuda.set_device(0)
    specs = W.config_specs(args.config)
    inputs = W.make_inputs_many(specs)
    ctx = svp.Context(num_gpus=1, device_ids=[0], profile_level=args.profile, arena_bytes=8 << 30,
                      max_chunks=args.max_chunks, streams_per_gpu=args.streams)
    vs = VPSet(ctx, specs, inputs, "host")
    jobs = svp.JobBatch(vs.job_list())
    import time
    walls, firsts = [], []
    for _ in range(args.reps):
        t0 = time.perf_counter()
        ctx.submit_batch(jobs)
        ctx.flush()
        walls.append((time.perf_counter() - t0) * 1e3)
        if args.profile:
            ops_r = ctx.plan()
            k = [o for o in ops_r if o["kind"] == svp.OP_KERNEL][:3]
            firsts.append([(o["stream"], round(o["measured_start_ns"] / 1e6, 2)) for o in k])
    st = ctx.flush_stats()
    if not args.profile:
        print(json.dumps({"config": args.config, "max_chunks": args.max_chunks, "streams": args.streams,
                          "profile": 0, "wall_ms": walls,
                          "max_connections": os.environ.get("CUDA_DEVICE_MAX_CONNECTIONS")}), flush=True)
        ctx.close()
        return
    ops = ctx.plan()
    h2d = [(o["measured_start_ns"], o["measured_start_ns"] + o["measured_ns"]) for o in ops if o["kind"] == svp.OP_H2D]
    d2h = [(o["measured_start_ns"], o["measured_start_ns"] + o["measured_ns"]) for o in ops if o["kind"] == svp.OP_D2H]
    ker = [(o["measured_start_ns"], o["measured_start_ns"] + o["measured_ns"]) for o in ops
           if o["kind"] == svp.OP_KERNEL]
    span = max(e for _, e in h2d + d2h + ker)
    hb = sum(o["bytes"] for o in ops if o["kind"] == svp.OP_H2D)
    db = sum(o["bytes"] for o in ops if o["kind"] == svp.OP_D2H)
    h_busy, d_busy = union_len(h2d), union_len(d2h)
    both = intersect_len(sorted(h2d), sorted(d2h))
    first_h2d_end = min(e for _, e in h2d) if h2d else 0.0
    last_h2d_end = max(e for _, e in h2d) if h2d else 0.0
    gaps = []
    hs = sorted(h2d)
    for (s0, e0), (s1, e1) in zip(hs, hs[1:]):
        if s1 > e0:
            gaps.append(s1 - e0)
    res = {"config": args.config, "max_chunks": args.max_chunks, "chunks": int(st["chunks"]), "wall_ms": walls,
           "first_kernels_per_flush": firsts,
           "streams": args.streams, "max_connections": os.environ.get("CUDA_DEVICE_MAX_CONNECTIONS"),
           "span_ms": span / 1e6, "host_total_ms": st["host_total_ns"] / 1e6,
           "h2d_bytes": hb, "d2h_bytes": db,
           "h2d_busy_ms": h_busy / 1e6, "d2h_busy_ms": d_busy / 1e6, "both_busy_ms": both / 1e6,
           "h2d_gbs_while_busy": hb / h_busy if h_busy else None, "d2h_gbs_while_busy": db / d_busy if d_busy else None,
           "h2d_gap_ms": sum(gaps) / 1e6, "h2d_gaps": len(gaps),
           "tail_after_last_h2d_ms": (span - last_h2d_end) / 1e6, "first_h2d_ms": first_h2d_end / 1e6,
           "kernel_busy_ms": union_len(ker) / 1e6,
           "ops": [{"i": i, "kind": o["kind"], "kernel": o["kernel"], "stream": o["stream"], "nvps": o["nvps"],
                    "bytes": o["bytes"], "start_ms": o["measured_start_ns"] / 1e6, "ms": o["measured_ns"] / 1e6,
                    "waits": o["waits"], "est_ms": o["est_ns"] / 1e6}
                   for i, o in enumerate(ops)]}
    print(json.dumps({k: v for k, v in res.items() if k != "ops"}), flush=True)
    if args.out:
        with open(args.out, "w") as f:
            json.dump(res, f, indent=1)
    ctx.close()


if __name__ == "__main__":
    main()
