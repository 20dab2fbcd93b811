"""Host logic of the hot path on CPU (dry-run contexts: no CUDA call at all).

Kernel Match, Job Dispatcher and Re-scheduler decisions are read back through
svp_plan_get and checked against oracle.sched (Johnson's rule, flow-shop makespan,
LPT) and against the invariants the paper states (identical kernels coalesced,
per-VP order kept, results divided back per VP)."""
import itertools
from collections import defaultdict

import numpy as np
import pytest

from oracle import sched
from paper_conf_dac_jungc15_b200 import svp

FAKE = 0x7F0000000000
KIND = {"vecadd": 3, "saxpy": 2, "hist256": 2, "blackscholes": 5, "sgemm": 3}


def fake_bufs(kernel, n=0, M=0, N=0, K=0, mem=svp.MEM_DEVICE, vp=0):
    base = FAKE + vp * (1 << 34)
    if kernel == "vecadd":
        return [(base, 4 * n, 1, mem), (base + 2**32, 4 * n, 1, mem), (base + 2**33, 4 * n, 2, mem)]
    if kernel == "saxpy":
        return [(base, 4 * n, 1, mem), (base + 2**32, 4 * n, 3, mem)]
    if kernel == "hist256":
        return [(base, n, 1, mem), (base + 2**32, 1024, 2, mem)]
    if kernel == "blackscholes":
        return [(base + i * 2**31, 4 * n, 1 if i < 3 else 2, mem) for i in range(5)]
    if kernel == "sgemm":
        return [(base, 4 * M * K, 1, mem), (base + 2**32, 4 * K * N, 1, mem), (base + 2**33, 4 * M * N, 2, mem)]


def args_for(kernel, n=0, M=0, N=0, K=0):
    return {"vecadd": lambda: svp.args_vecadd(n), "saxpy": lambda: svp.args_saxpy(n, 2.0),
            "hist256": lambda: svp.args_hist256(n), "blackscholes": lambda: svp.args_blackscholes(n, 0.02, 0.3),
            "sgemm": lambda: svp.args_sgemm(M, N, K)}[kernel]()


def submit(c, vp, kernel, n=0, M=0, N=0, K=0, mem=svp.MEM_DEVICE):
    kid = c.kernel(kernel)
    return c.submit(vp, kid, args_for(kernel, n, M, N, K), fake_bufs(kernel, n, M, N, K, mem, vp))


MIX = ("vecadd", "saxpy", "hist256", "blackscholes")


def test_kernel_match_groups_identical_kernels():
    with svp.Context(dry_run=True) as c:
        for vp in range(64):
            submit(c, vp, MIX[vp % 4], n=1000 + 37 * vp)  # ragged sizes are still "identical"
        c.flush()
        ops = c.plan()
        st = c.flush_stats()
        assert st["groups"] == 4 and st["launches"] == 4
        seen = set()
        for op in ops:
            assert op["kind"] == svp.OP_KERNEL and op["nvps"] == 16
            assert op["vps"] == sorted(op["vps"])                    # members in VP order (R12)
            kname = [k for k in MIX if c.kernel_ids[k] == op["kernel"]][0]
            assert all(MIX[v % 4] == kname for v in op["vps"])
            seen |= set(op["vps"])
        assert seen == set(range(64))


def test_ragged_gemm_shapes_share_one_launch():
    """Reading R1 as revised for NEXT item f2: GEMMs of different (M, N, K) are identical
    kernel requests too -- one grouped launch carries every VP's shape in its tile table."""
    with svp.Context(dry_run=True) as c:
        for vp in range(6):
            s = 128 if vp < 4 else 256
            submit(c, vp, "sgemm", M=s, N=s + 64, K=s // 2)
        c.flush()
        ops = c.plan()
        assert [op["nvps"] for op in ops] == [6]
        assert ops[0]["flops"] == sum(2.0 * s * (s + 64) * (s // 2) for s in [128] * 4 + [256] * 2)


@pytest.mark.parametrize("impl", [svp.SGEMM_TF32BF16, svp.SGEMM_3XTF32, svp.SGEMM_FFMA])
def test_sgemm_accuracy_routing_chunked(impl):
    """DESIGN R23, sgemm_kchunk = 512 (strict mode): with K-chunked accumulation a beta == 0
    "sgemm" job stays on the tensor cores at any K; a beta != 0 job (not chunked) past one
    chunk matches apart and runs on FFMA.  With FFMA every job coalesces into one launch."""
    with svp.Context(dry_run=True, sgemm_impl=impl, sgemm_kchunk=512) as c:
        # the beta != 0 chunk limit: 512 k for TF32+2xBF16, 256 k for 3xTF32
        lim = 256 if impl == svp.SGEMM_3XTF32 else 512
        jobs = [(512, 0.0), (4096, 0.0), (lim, 1.0), (lim + 4, 1.0), (8192, 0.5)]
        kid = c.kernel("sgemm")
        for vp, (K, beta) in enumerate(jobs):
            bufs = fake_bufs("sgemm", M=256, N=256, K=K, vp=vp)
            bufs[0] = (bufs[0][0], 4 * 256 * 8192, bufs[0][2], bufs[0][3])  # room for every K
            bufs[1] = (bufs[1][0], 4 * 256 * 8192, bufs[1][2], bufs[1][3])
            if beta:
                bufs[2] = (bufs[2][0], bufs[2][1], svp.DIR_INOUT, bufs[2][3])
            c.submit(vp, kid, svp.args_sgemm(256, 256, K, 1.0, beta), bufs)
        c.flush()
        sg = [op for op in c.plan() if op["kind"] == svp.OP_KERNEL]
        groups = sorted(sorted(op["vps"]) for op in sg)
        if impl == svp.SGEMM_FFMA:
            assert groups == [[0, 1, 2, 3, 4]]
        else:
            assert groups == [[0, 1, 2], [3, 4]]


@pytest.mark.parametrize("impl,kmax", [(svp.SGEMM_TF32BF16, 2048), (svp.SGEMM_3XTF32, 1024), (svp.SGEMM_FFMA, None)])
def test_sgemm_accuracy_routing_unchunked(impl, kmax):
    """DESIGN R23, sgemm_kchunk = 0 (one accumulation per tile): jobs with K above the measured
    limit of the split's single accumulation (2048 for TF32+2xBF16, 1024 for 3xTF32) match
    apart and run on FFMA."""
    with svp.Context(dry_run=True, sgemm_impl=impl, sgemm_kchunk=0) as c:
        Ks = [512, 1024, 2048, 2052, 4096]
        for vp, K in enumerate(Ks):
            submit(c, vp, "sgemm", M=256, N=256, K=K)
        c.flush()
        sg = [op for op in c.plan() if op["kind"] == svp.OP_KERNEL]
        if kmax is None:
            assert len(sg) == 1 and sg[0]["nvps"] == 5
        else:
            groups = sorted(sorted(op["vps"]) for op in sg)
            want = sorted([[v for v, K in enumerate(Ks) if K <= kmax], [v for v, K in enumerate(Ks) if K > kmax]])
            assert groups == want


def test_sgemm_kchunk_must_be_a_multiple_of_16():
    for bad in (-16, 8, 100):
        with pytest.raises(svp.SvpError):
            svp.Context(dry_run=True, sgemm_kchunk=bad)


def test_no_coalescing_is_one_launch_per_job_in_submission_order():
    with svp.Context(dry_run=True, coalesce=False, interleave=False) as c:
        order = [5, 3, 9, 1]
        for vp in order:
            submit(c, vp, "vecadd", n=100)
        c.flush()
        ops = c.plan()
        assert [op["vps"] for op in ops] == [[v] for v in order]
        assert all(op["stream"] == 0 for op in ops)


def test_program_order_levels_and_dependencies():
    with svp.Context(dry_run=True) as c:
        for vp in range(8):
            submit(c, vp, "vecadd", n=10000, mem=svp.MEM_HOST_PINNED)
            submit(c, vp, "saxpy", n=20000, mem=svp.MEM_HOST_PINNED)
            submit(c, vp, "hist256", n=30000, mem=svp.MEM_HOST_PINNED)
        c.flush()
        ops = c.plan()
        assert c.flush_stats()["levels"] == 3
        per_vp = defaultdict(list)
        for i, op in enumerate(ops):
            for v in op["vps"]:
                per_vp[v].append((i, op))
        for v, lst in per_vp.items():
            levels = [op["level"] for _, op in lst]
            assert levels == sorted(levels)
            # every op of level l starts after every op of level l-1 of the same VP ends
            for (_, a), (_, b) in itertools.combinations(lst, 2):
                if b["level"] > a["level"]:
                    assert b["sim_start_ns"] >= a["sim_end_ns"] - 1e-6


def test_sparse_vp_ids_plan_like_compact_ids():
    """The planner keeps per-VP state in a flat array for compact VP ids and in a hash map
    for sparse ones (ids up to 2^20): both must give the same plan for the same program."""
    def plan_for(ids):
        with svp.Context(dry_run=True) as c:
            for rep in range(2):
                for k, vp in enumerate(ids):
                    submit(c, vp, MIX[(k + rep) % 4], n=5000 + 100 * k, mem=svp.MEM_HOST_PINNED)
            c.flush()
            inv = {v: i for i, v in enumerate(ids)}
            return [(op["kind"], op["level"], op["kernel"], sorted(inv[v] for v in op["vps"]), op["stream"],
                     round(op["sim_start_ns"], 3)) for op in c.plan()], c.flush_stats()["levels"]
    sparse = [5, (1 << 20) - 1, 300000, 77, 123456, 999999]
    compact = [0, 5, 3, 1, 2, 4]  # the ranks of the sparse ids (same relative order)
    ps, ls = plan_for(sparse)
    pc, lc = plan_for(compact)
    assert ls == lc == 2
    assert ps == pc


def _host_cfg_plan(c, nvps=32, n=1 << 20):
    for vp in range(nvps):
        submit(c, vp, MIX[vp % 4], n=n + 4096 * vp, mem=svp.MEM_HOST_PINNED)
    c.flush()
    return c.plan()


def test_interleaving_streams_and_chunks():
    S = 4
    with svp.Context(dry_run=True, streams_per_gpu=S) as c:
        ops = _host_cfg_plan(c)
        st = c.flush_stats()
        assert st["chunks"] > st["groups"]          # groups split for copy/compute overlap
        kinds = defaultdict(set)
        for op in ops:
            kinds[op["kind"]].add(op["stream"])
        assert kinds[svp.OP_H2D] == {S} and kinds[svp.OP_D2H] == {S + 1}
        assert kinds[svp.OP_KERNEL] <= set(range(S)) and len(kinds[svp.OP_KERNEL]) > 1
        # chunks of a group partition its members, contiguous in VP order
        by_group = defaultdict(list)
        for op in ops:
            if op["kind"] == svp.OP_KERNEL:
                by_group[op["group"]].append((op["chunk"], op["vps"]))
        for g, chunks in by_group.items():
            members = [v for _, vs in sorted(chunks) for v in vs]
            assert members == sorted(members) and len(set(members)) == len(members)
        assert st["sim_makespan_ns"] < st["sim_serial_ns"]


def _chunk_triples(ops):
    t = {}
    for op in ops:
        key = (op["group"], op["chunk"])
        t.setdefault(key, [0.0, 0.0, 0.0])
        t[key][{svp.OP_H2D: 0, svp.OP_KERNEL: 1, svp.OP_D2H: 2}[op["kind"]]] = op["est_ns"]
    return t


def test_johnson_order_matches_oracle():
    with svp.Context(dry_run=True) as c:
        ops = _host_cfg_plan(c)
        trip = _chunk_triples(ops)
        canon = sorted(trip)                                   # (group, chunk) order = tie-break order
        jobs = [tuple(trip[k]) for k in canon]
        want = [canon[i] for i in sched.johnson_order(jobs)]
        got = [(op["group"], op["chunk"]) for op in ops if op["kind"] == svp.OP_KERNEL]
        assert got == want


def test_simulated_makespan_is_flowshop_of_plan_order():
    with svp.Context(dry_run=True) as c:
        ops = _host_cfg_plan(c)
        trip = _chunk_triples(ops)
        order = [(op["group"], op["chunk"]) for op in ops if op["kind"] == svp.OP_KERNEL]
        jobs = [tuple(trip[k]) for k in order]
        assert all(a > 0 and b > 0 and cc > 0 for a, b, cc in jobs)
        ms = c.flush_stats()["sim_makespan_ns"]
        assert ms == pytest.approx(sched.flowshop_makespan(jobs), rel=1e-12)
        assert c.flush_stats()["sim_serial_ns"] == pytest.approx(sched.serial_time(jobs), rel=1e-12)
        if len(jobs) <= 7:
            assert ms >= sched.best_makespan(jobs) - 1e-6


@pytest.mark.parametrize("seed", range(6))
def test_johnson_plan_optimal_when_copy_bound(seed):
    """Small host-resident mixes built to be PCIe-bound (Tk << Tin, Tout: vecadd / SAXPY /
    Black-Scholes of >= 1 Mi elements, whose copies are ~8-16 B/elem at PCIe speed against
    12-20 B/elem at HBM speed) -- Johnson's 3-machine condition holds on every seed (asserted,
    so the test is never vacuous), and then the planned order is optimal (brute force over
    all orders)."""
    g = np.random.default_rng(seed)
    kinds = ("vecadd", "saxpy", "blackscholes")
    with svp.Context(dry_run=True, max_chunks=1) as c:
        for vp in range(int(g.integers(2, 7))):
            submit(c, vp, kinds[int(g.integers(0, 3))], n=int(g.integers(10, 40)) * 100000, mem=svp.MEM_HOST_PINNED)
        c.flush()
        ops = c.plan()
        trip = _chunk_triples(ops)
        jobs = [tuple(v) for v in trip.values()]
        assert min(j[0] for j in jobs) >= max(j[1] for j in jobs) or min(j[2] for j in jobs) >= max(j[1] for j in jobs)
        assert c.flush_stats()["sim_makespan_ns"] == pytest.approx(sched.best_makespan(jobs), rel=1e-9)


def test_dispatcher_shards_vps_across_gpus():
    with svp.Context(dry_run=True, num_gpus=4) as c:
        kids = [c.kernel(k) for k in MIX]
        vps = list(range(64))
        costs = [1000.0 + (v * 7919) % 97 for v in vps]
        devs = c.assign_vps(vps, [kids[v % 4] for v in vps], costs)
        for k in range(4):
            cnt = np.bincount([devs[v] for v in vps if v % 4 == k], minlength=4)
            assert cnt.max() - cnt.min() <= 1                 # every GPU gets its share of every class
        assert all(c.vp_device(v) == devs[v] for v in vps)   # sticky
        for vp in vps:
            submit(c, vp, MIX[vp % 4], n=5000)
        c.flush()
        for op in c.plan():
            assert all(devs[v] == op["device"] for v in op["vps"])
        assert c.flush_stats()["launches"] == 16              # 4 kernels x 4 GPUs


def test_lpt_single_class_matches_oracle_and_graham():
    g = np.random.default_rng(3)
    for G in (2, 3, 4, 8):
        for _ in range(10):
            costs = list(map(float, g.integers(1, 100, int(g.integers(1, 9)))))
            got = svp.lpt_partition([7] * len(costs), costs, G)
            assert got == sched.lpt_partition(costs, G)
            if G <= 3:
                opt = sched.best_partition_makespan(costs, G)
                assert sched.partition_makespan(costs, got, G) <= sched.graham_bound(G) * opt + 1e-9


def test_arena_ring_reuse_waits():
    # host-resident jobs larger in total than the arena: slots must be reused, and the
    # reusing H2D must start after the D2H that frees the slot
    with svp.Context(dry_run=True, arena_bytes=64 << 20, max_chunks=4) as c:
        for vp in range(16):
            submit(c, vp, "vecadd", n=1 << 20, mem=svp.MEM_HOST_PINNED)  # 12 MiB staged per job
        c.flush()
        ops = c.plan()
        assert c.flush_stats()["chunks"] >= 4
        h2d = [op for op in ops if op["kind"] == svp.OP_H2D]
        d2h = [op for op in ops if op["kind"] == svp.OP_D2H]
        assert sum(op["bytes"] for op in h2d) == 16 * 8 * (1 << 20)
        assert sum(op["bytes"] for op in d2h) == 16 * 4 * (1 << 20)


def _arena_order_violations(ops):
    """Pairs of chunks whose staging-arena ranges overlap where the later chunk's first op
    is not ordered after the earlier chunk's last op (its release).  Order = the plan's
    event waits plus issue order on each (device, stream)."""
    chunks = []  # (device, first op, last op, off, len) in issue order
    for i, op in enumerate(ops):
        key = (op["device"], op["group"], op["chunk"])
        if chunks and chunks[-1][0] == key:
            chunks[-1][2] = i
        else:
            chunks.append([key, i, i, op["arena_off"], op["arena_len"]])
    succ = defaultdict(set)
    last_on = {}
    for i, op in enumerate(ops):
        for w in op["waits"]:
            succ[w].add(i)
        s = (op["device"], op["stream"])
        if s in last_on:
            succ[last_on[s]].add(i)
        last_on[s] = i

    def reaches(a, b):
        seen, todo = {a}, [a]
        while todo:
            x = todo.pop()
            if x == b:
                return True
            for y in succ[x]:
                if y not in seen and y <= b:
                    seen.add(y)
                    todo.append(y)
        return False

    bad = []
    for p in range(len(chunks)):
        kp, fp, lp, op_, lnp = chunks[p]
        if not lnp:
            continue
        for q in range(p + 1, len(chunks)):
            kq, fq, lq, oq, lnq = chunks[q]
            if not lnq or kq[0] != kp[0]:
                continue
            if op_ < oq + lnq and oq < op_ + lnp and not reaches(lp, fq):
                bad.append((kp, kq))
    return bad


def test_arena_wrap_mixed_residency_orders_every_overlap():
    """a small arena that wraps, chunks whose only staged buffer is an OUTPUT
    (their first op is the kernel, not an H2D on the shared copy stream), mixed
    DEVICE / HOST_PINNED buffers per job, two program-order levels.  Every later chunk
    placed over an earlier chunk's arena bytes must start after that chunk's last op."""
    H, D = svp.MEM_HOST_PINNED, svp.MEM_DEVICE
    # the advisor's layout: X = saxpy (staged), A = vecadd, B = hist256 wraps to 0, then a
    # level-1 vecadd whose only staged buffer is its output lands inside A's region
    with svp.Context(dry_run=True, arena_bytes=2 << 20, max_chunks=1, interleave=True) as c:
        kid = {k: c.kernel(k) for k in MIX}
        n = 40000
        bufs_x = [(FAKE, 4 * n, 1, H), (FAKE + 2**32, 4 * n, 3, H)]                     # 320 KB staged
        bufs_a = [(FAKE + 2**34, 4 * n * 2, 1, H), (FAKE + 2**35, 4 * n * 2, 1, H), (FAKE + 2**36, 4 * n * 2, 2, H)]
        bufs_b = [(FAKE + 2**37, 300000, 1, D), (FAKE + 2**38, 1024, 2, H)]          # counts only staged
        c.submit(0, kid["saxpy"], svp.args_saxpy(n, 2.0), bufs_x)
        c.submit(1, kid["vecadd"], svp.args_vecadd(2 * n), bufs_a)
        c.submit(2, kid["hist256"], svp.args_hist256(300000), bufs_b)
        c.submit(2, kid["hist256"], svp.args_hist256(300000), bufs_b)
        c.submit(3, kid["vecadd"], svp.args_vecadd(2 * n),
                 [(FAKE + 2**39, 8 * n, 1, D), (FAKE + 2**40, 8 * n, 1, D), (FAKE + 2**41, 8 * n, 2, H)])
        c.submit(3, kid["vecadd"], svp.args_vecadd(2 * n),
                 [(FAKE + 2**39, 8 * n, 1, D), (FAKE + 2**40, 8 * n, 1, D), (FAKE + 2**41, 8 * n, 2, H)])
        c.flush()
        ops = c.plan()
        assert any(op["arena_len"] for op in ops)
        assert _arena_order_violations(ops) == []


# seeds 30, 111, 113, 117, 179, 185 and 198 each produced an unordered overlap with the
# round-1 planner (overlapped slots were dropped from the in-flight list)
@pytest.mark.parametrize("seed", [30, 111, 113, 117, 179, 185, 198] + list(range(8)))
def test_arena_wrap_random_mixes_have_no_unordered_overlap(seed):
    g = np.random.default_rng(seed)
    H, D = svp.MEM_HOST_PINNED, svp.MEM_DEVICE
    arena = int(g.integers(1, 5)) << 20
    with svp.Context(dry_run=True, arena_bytes=arena, max_chunks=int(g.integers(1, 5)),
                     streams_per_gpu=int(g.integers(1, 4)), num_gpus=int(g.integers(1, 3))) as c:
        for vp in range(int(g.integers(4, 24))):
            for _ in range(int(g.integers(1, 4))):
                k = MIX[int(g.integers(0, 4))]
                n = int(g.integers(1, 120000))
                bufs = fake_bufs(k, n=n, vp=vp)
                bufs = [(p, b, d, H if g.random() < 0.5 else D) for (p, b, d, _m) in bufs]
                c.submit(vp, c.kernel(k), args_for(k, n=n), bufs)
        try:
            c.flush()
        except svp.SvpError as e:  # a job larger than half the arena: SVP_E_NOMEM, nothing planned
            assert e.status == svp.SVP_E_NOMEM
            return
        ops = c.plan()
        assert _arena_order_violations(ops) == []


def test_job_larger_than_arena_is_nomem():
    with svp.Context(dry_run=True, arena_bytes=1 << 20) as c:
        submit(c, 0, "vecadd", n=1 << 20, mem=svp.MEM_HOST_PINNED)
        with pytest.raises(svp.SvpError) as e:
            c.flush()
        assert e.value.status == svp.SVP_E_NOMEM


# ---------------------------------------------------------------- NEXT f4 (host side)
def test_hetero_merges_elementwise_groups_only():
    """cfg hetero: vecadd / SAXPY / Black-Scholes of one (level, GPU) form ONE group with
    kernel id SVP_KERNEL_EW_MIX, members in VP order; hist256 and SGEMM keep their own."""
    kinds = ("vecadd", "saxpy", "hist256", "blackscholes", "sgemm")
    with svp.Context(dry_run=True, hetero=True) as c:
        for vp in range(40):
            k = kinds[vp % 5]
            if k == "sgemm":
                submit(c, vp, k, M=128, N=128, K=64)
            else:
                submit(c, vp, k, n=5000 + 911 * vp)
        c.flush()
        ops = c.plan()
        st = c.flush_stats()
        assert st["groups"] == 3 and st["launches"] == 3
        by_kernel = {op["kernel"]: op for op in ops}
        mix = by_kernel[svp.KERNEL_EW_MIX]
        assert mix["vps"] == sorted(v for v in range(40) if kinds[v % 5] in ("vecadd", "saxpy", "blackscholes"))
        assert by_kernel[c.kernel_ids["hist256"]]["nvps"] == 8
        assert by_kernel[c.kernel_ids["sgemm"]]["nvps"] == 8


def test_hetero_keeps_program_order_levels():
    with svp.Context(dry_run=True, hetero=True) as c:
        for vp in range(6):
            submit(c, vp, "vecadd", n=1000)
            submit(c, vp, "saxpy", n=1000)
        c.flush()
        ops = c.plan()
        assert [op["level"] for op in ops] == [0, 1]
        assert all(op["kernel"] == svp.KERNEL_EW_MIX and op["nvps"] == 6 for op in ops)


def test_graph_mode_reuses_identical_plans():
    """cfg graph: a flush with the same requests as the previous one reuses its plan
    (same ops, streams, order); any change in the requests replans."""
    with svp.Context(dry_run=True, graph=True) as c:
        def round_(n0):
            for vp in range(12):
                submit(c, vp, MIX[vp % 4], n=n0 + 100 * vp, mem=svp.MEM_HOST_PINNED)
            c.flush()
            return c.plan(), c.flush_stats()
        p1, s1 = round_(100000)
        p2, s2 = round_(100000)
        p3, s3 = round_(100001)
        assert s1["plan_reused"] == 0 and s2["plan_reused"] == 1 and s3["plan_reused"] == 0
        strip = lambda p: [{k: v for k, v in op.items() if k != "measured_ns"} for op in p]
        assert strip(p1) == strip(p2)
        assert s2["sim_makespan_ns"] == s1["sim_makespan_ns"]
        assert strip(p3) != strip(p1)


def test_plan_cache_alternating_request_sets():
    """cfg graph (the default): the plans of the last 32 flushes before the previous one are
    cached too, so a loop that rotates buffer sets reuses one plan per set; a set not seen
    within the last 33 flushes is planned afresh.  A reused plan equals the original."""
    with svp.Context(dry_run=True) as c:
        def flush_set(k):
            for vp in range(6):
                submit(c, vp, MIX[vp % 4], n=50000 + 1000 * k + vp, mem=svp.MEM_DEVICE)
            c.flush()
            strip = [{kk: v for kk, v in op.items() if kk != "measured_ns"} for op in c.plan()]
            return c.flush_stats()["plan_reused"], strip
        first = {k: flush_set(k)[1] for k in range(3)}
        for k in (0, 1, 2, 0, 2, 1):
            reused, plan = flush_set(k)
            assert reused == 1 and plan == first[k], k
        for k in range(3, 37):  # 34 new sets: 0, 1, 2 fall out of the cache
            assert flush_set(k)[0] == 0
        assert flush_set(0)[0] == 0
        assert flush_set(10)[0] == 1


def test_graph_mode_off_never_reuses():
    with svp.Context(dry_run=True, graph=False) as c:
        for _ in range(2):
            submit(c, 0, "vecadd", n=1000)
            c.flush()
        assert c.flush_stats()["plan_reused"] == 0
