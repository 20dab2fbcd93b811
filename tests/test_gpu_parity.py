"""GPU parity: every VP's output from the coalesced / interleaved sm_100a path equals
the oracle (bit-exact for integer-like kernels, stated tolerance for fp32), through
the C-ABI, for device- and host-resident buffers, serial and coalesced modes."""
import dataclasses

import numpy as np
import pytest
import torch

import oracle
import workloads as W
from gpu_common import check_job, inputs_for, run_svp
from paper_conf_dac_jungc15_b200 import svp
from paper_conf_dac_jungc15_b200.vpset import VPSet

pytestmark = pytest.mark.gpu

MODES = {
    "coalesced_interleaved": dict(coalesce=True, interleave=True),
    "coalesced_1stream": dict(coalesce=True, interleave=False),
    "serial_sync": dict(coalesce=False, interleave=False, sync_each_job=True),
}


@pytest.fixture(scope="module")
def cfg5_sgemm_oracle():
    """cfg5 inputs and the oracle's full products of 4 of its 51 SGEMM 2048^3 VPs (first,
    last, two middle; one VP per host thread, ~10 s)."""
    specs = W.config_specs(5)
    inputs = W.make_inputs_many(specs)
    sg = [i for i, s in enumerate(specs) if s.kernel == "sgemm"]
    pick = [sg[0], sg[len(sg) // 3], sg[2 * len(sg) // 3], sg[-1]]
    want = oracle.run_jobs([specs[i] for i in pick], [inputs[i] for i in pick], threads=4)
    return specs, inputs, pick, want


@pytest.fixture(scope="module")
def small():
    specs = W.mixed_small(nvps=30, max_n=70000)
    return specs, inputs_for(specs)


@pytest.mark.parametrize("mode", list(MODES))
@pytest.mark.parametrize("residency", ["device", "host"])
def test_mixed_small(small, mode, residency):
    specs, inputs = small
    outs, prof, st = run_svp(specs, inputs, residency, **MODES[mode])
    for s, inp, got in zip(specs, inputs, outs):
        check_job(s, inp, got)
    if mode == "serial_sync":
        assert st["launches"] == len(specs)   # one launch op per job, no coalescing
    else:
        assert st["groups"] < len(specs)


def test_coalesced_bit_identical_to_serial(small):
    """T5: the same kernel code on one segment or many gives identical bits (per-element /
    per-tile op order does not depend on coalescing)."""
    specs, inputs = small
    a, _, _ = run_svp(specs, inputs, "device", coalesce=True)
    b, _, _ = run_svp(specs, inputs, "device", coalesce=False, interleave=False)
    for s, x, y in zip(specs, a, b):
        for k in x:
            assert np.array_equal(x[k].view(np.uint32) if x[k].dtype == np.float32 else x[k],
                                  y[k].view(np.uint32) if y[k].dtype == np.float32 else y[k]), (s.vp, s.kernel, k)


@pytest.mark.parametrize("residency", ["device", "host"])
def test_config4_ragged_full_size(residency):
    """BASELINE config 4: 64 VPs, ragged 64Ki..16Mi + adversarial sizes, misaligned views."""
    specs = W.config_specs(4)
    for s in specs[8:16]:
        s.misalign = 2 if s.vp % 2 else 1
    inputs = inputs_for(specs)
    outs, _, st = run_svp(specs, inputs, residency)
    assert st["groups"] == 4
    want = oracle.run_jobs(specs, inputs)
    for s, inp, got, w in zip(specs, inputs, outs, want):
        check_job(s, inp, got, w)


def test_config3_interleaved_host():
    specs = W.config_specs(3, scale=4)
    inputs = inputs_for(specs)
    outs, prof, st = run_svp(specs, inputs, "host", profile_level=1)
    assert st["chunks"] > st["groups"]
    want = oracle.run_jobs(specs, inputs)
    for s, inp, got, w in zip(specs, inputs, outs, want):
        check_job(s, inp, got, w)


@pytest.mark.parametrize("impl", [svp.SGEMM_FFMA, svp.SGEMM_3XTF32])
@pytest.mark.parametrize("int_inputs", [True, False])
def test_config2_sgemm_512(int_inputs, impl):
    specs = W.config_specs(2, sgemm_int=int_inputs)
    inputs = inputs_for(specs)
    outs, _, st = run_svp(specs, inputs, "device", sgemm_impl=impl)
    assert st["launches"] == 1
    want = oracle.run_jobs(specs, inputs)
    for s, inp, got, w in zip(specs, inputs, outs, want):
        check_job(s, inp, got, w)


@pytest.mark.parametrize("impl", [svp.SGEMM_FFMA, svp.SGEMM_3XTF32])
def test_sgemm_alpha_beta_ragged_edges(impl):
    specs = []
    for v, (M, N, K) in enumerate([(200, 136, 40), (200, 136, 40), (1, 4, 4), (129, 260, 0), (64, 68, 1000)]):
        specs.append(W.JobSpec(v, "sgemm", M=M, N=N, K=K, alpha=1.5, beta=-0.5))
    inputs = inputs_for(specs)
    outs, _, _ = run_svp(specs, inputs, "device", sgemm_impl=impl)
    for s, inp, got in zip(specs, inputs, outs):
        check_job(s, inp, got)


def test_program_order_chain():
    """A VP's jobs run in program order: vecadd writes c, then SAXPY reads c as x and
    updates y in place, then SAXPY again -- one flush."""
    n = 100003
    ctx = svp.Context(num_gpus=1)
    va, sx = ctx.register_kernel("vecadd"), ctx.register_kernel("saxpy")
    jobs, expect, bufs = [], [], []
    for vp in range(6):
        g = W.rng(9, vp, 1)
        a, b, y = (W.uniform_f32(g, n, -1, 1) for _ in range(3))
        ta, tb, ty = (torch.from_numpy(x).cuda() for x in (a, b, y))
        tc = torch.empty_like(ta)
        bufs.append((ta, tb, tc, ty))
        c = oracle.vecadd(a, b)
        y1 = oracle.saxpy(0.5 + vp, c, y)
        y2 = oracle.saxpy(-2.0, c, y1)
        expect.append((c, y2))
        p = lambda t: t.data_ptr()
        jobs.append((vp, va, svp.args_vecadd(n), [(p(ta), 4 * n, 1, 0), (p(tb), 4 * n, 1, 0), (p(tc), 4 * n, 2, 0)]))
        jobs.append((vp, sx, svp.args_saxpy(n, 0.5 + vp), [(p(tc), 4 * n, 1, 0), (p(ty), 4 * n, 3, 0)]))
        jobs.append((vp, sx, svp.args_saxpy(n, -2.0), [(p(tc), 4 * n, 1, 0), (p(ty), 4 * n, 3, 0)]))
    ctx.submit_batch(jobs)
    ctx.flush()
    assert ctx.flush_stats()["levels"] == 3
    for (ta, tb, tc, ty), (c, y2) in zip(bufs, expect):
        assert np.array_equal(tc.cpu().numpy(), c)
        assert np.array_equal(ty.cpu().numpy(), y2)
    ctx.close()


def test_profiler_conservation_and_kernel_stats(small):
    specs, inputs = small
    ctx = svp.Context(num_gpus=1, profile_level=1)
    vs = VPSet(ctx, specs, inputs, "host")
    vs.submit()
    ctx.flush()
    ops = ctx.plan()
    tot = ctx.profile(-1)
    per = [ctx.profile(s.vp) for s in specs]
    k_meas = sum(op["measured_ns"] for op in ops if op["kind"] == svp.OP_KERNEL)
    h_meas = sum(op["measured_ns"] for op in ops if op["kind"] == svp.OP_H2D)
    assert all(op["measured_ns"] >= 0 for op in ops)
    assert sum(p["kernel_ns"] for p in per) == pytest.approx(k_meas, rel=1e-9)
    assert sum(p["h2d_ns"] for p in per) == pytest.approx(h_meas, rel=1e-9)
    assert tot["kernel_ns"] == pytest.approx(k_meas, rel=1e-9)
    assert sum(p["jobs"] for p in per) == len(specs)
    n_launch = sum(ctx.kernel_stats(k)["launches"] for k in vs.kids.values())
    assert n_launch == sum(1 for op in ops if op["kind"] == svp.OP_KERNEL)
    st = ctx.flush_stats()
    assert 0 < st["device_ns"] <= st["host_total_ns"]
    ctx.close()


def test_profiler_measured_split_level2():
    """profile_level 2 (a10 second opinion): a segment launch's event-timed duration is
    split over its VPs by the SM cycles measured on their tiles.  Outputs stay exact, the
    split conserves the launch time, and for full-tile VPs it agrees with the algorithmic
    byte split of level 1 (uniform work per tile) within 25 %."""
    sizes = [1 << 22, 1 << 20, (1 << 20) + 12345, 3 << 20]
    specs = [W.JobSpec(v, "vecadd", n=n) for v, n in enumerate(sizes)]
    specs += [W.JobSpec(4 + v, "hist256", n=n) for v, n in enumerate(sizes)]
    inputs = inputs_for(specs)
    shares = {}
    for level in (1, 2):
        ctx = svp.Context(num_gpus=1, profile_level=level)
        try:
            vs = VPSet(ctx, specs, inputs, "device")
            jb = svp.JobBatch(vs.job_list())
            ctx.submit_batch(jb)
            ctx.flush()
            ctx.reset_profile()
            for _ in range(3):
                ctx.submit_batch(jb)
                ctx.flush()
            torch.cuda.synchronize()
            for i, (sp, inp) in enumerate(zip(specs, inputs)):
                check_job(sp, inp, vs.output(i))
            per_vp = [ctx.profile(sp.vp)["kernel_ns"] for sp in specs]
            tot = ctx.profile(-1)["kernel_ns"]
            ks = sum(ctx.kernel_stats(ctx.kernel_ids[k])["total_ns"] for k in ("vecadd", "hist256"))
            assert abs(sum(per_vp) - tot) <= 1e-6 * tot and abs(tot - ks) <= 1e-6 * ks
            assert all(x > 0 for x in per_vp)
            shares[level] = per_vp
        finally:
            ctx.close()
    for lo, hi in ((0, 4), (4, 8)):
        s1 = np.array(shares[1][lo:hi]) / sum(shares[1][lo:hi])
        s2 = np.array(shares[2][lo:hi]) / sum(shares[2][lo:hi])
        assert np.all(np.abs(s2 / s1 - 1) < 0.25), (lo, s1, s2)


@pytest.mark.parametrize("hetero", [False, True])
def test_dynamic_tile_order_repeated(hetero):
    """A Black-Scholes (or mixed) launch alone on the GPU takes its tiles in dynamic order
    from a self-resetting counter pair: three flushes in a row, outputs poisoned with NaN
    before each, must all be recomputed and match the oracle (a counter left non-zero
    would make the next launch skip tiles)."""
    kinds = ("blackscholes", "vecadd", "saxpy") if hetero else ("blackscholes",)
    specs = [W.JobSpec(v, kinds[v % len(kinds)], n=(1 << 18) + 4097 * v, R=0.02, V=0.3, a=1.5) for v in range(9)]
    inputs = inputs_for(specs)
    ctx = svp.Context(num_gpus=1, hetero=hetero)
    try:
        vs = VPSet(ctx, specs, inputs, "device")
        jb = svp.JobBatch(vs.job_list())
        for r in range(3):
            vs.load_inputs()
            for i, sp in enumerate(specs):
                for name in ("call", "put", "c"):
                    if name in vs.bufs[i]:
                        vs.bufs[i][name].fill_(float("nan"))
            torch.cuda.synchronize()  # the fills run on torch's stream, the flush on libsvp's
            ctx.submit_batch(jb)
            ctx.flush()
            torch.cuda.synchronize()
            assert ctx.flush_stats()["launches"] == 1
            for i, (sp, inp) in enumerate(zip(specs, inputs)):
                check_job(sp, inp, vs.output(i))
    finally:
        ctx.close()


def test_profiler_split_vs_serial_per_vp_launches():
    """SURVEY §4 T9, against an independent measurement: the event-timed duration of each
    VP's OWN launch when the same jobs run uncoalesced (serial mode).  A standalone launch
    is not proportional to the VP's bytes -- it pays the launch and a partly filled last
    round of tiles, Eq 9's T_o + T_e * ceil(xi / lambda): 4 Mi elements took
    ~18 us against ~7 us of bandwidth -- which is exactly what coalescing amortises.  So the
    checks are: serial times rise with the VP's size; the coalesced launch takes less than
    the VP's serial launches together; and the level-1 shares (bytes) rank the VPs as their
    serial launches do, each within a factor 2 of the serial share.  The level-2 split
    (thread 0's cycles per tile) is only checked for conservation here: it weighs a tile by
    its latency when it ran, which depends on what else was in flight."""
    sizes = np.array([1 << 22, 2 << 22, 3 << 22, 4 << 22, 6 << 22])
    kinds = ("vecadd", "saxpy")
    nv = len(sizes)
    specs = [W.JobSpec(v, kinds[v // nv], n=int(sizes[v % nv]), a=1.25) for v in range(2 * nv)]
    inputs = inputs_for(specs)
    reps = 5

    def per_vp(**cfg):
        ctx = svp.Context(num_gpus=1, **cfg)
        try:
            vs = VPSet(ctx, specs, inputs, "device")
            jb = svp.JobBatch(vs.job_list())
            ctx.submit_batch(jb)
            ctx.flush()
            ctx.reset_profile()
            for _ in range(reps):
                ctx.submit_batch(jb)
                ctx.flush()
            torch.cuda.synchronize()
            return np.array([ctx.profile(sp.vp)["kernel_ns"] for sp in specs]) / reps
        finally:
            ctx.close()

    serial = per_vp(coalesce=False, interleave=False, profile_level=1)
    # one stream, so each coalesced launch's event-timed duration is its own
    coal = {level: per_vp(profile_level=level, interleave=False) for level in (1, 2)}
    for lo in (0, nv):  # per kernel class (one coalesced launch each)
        t = serial[lo:lo + nv]
        assert np.all(np.diff(t) > 0), (kinds[lo // nv], t)
        c = coal[1][lo:lo + nv]
        assert c.sum() < t.sum(), (kinds[lo // nv], c.sum(), t.sum())  # coalescing gain
        assert np.all(np.diff(c) > 0), (kinds[lo // nv], c)              # same ranking
        a, b = t / t.sum(), c / c.sum()
        assert np.all((b / a > 0.5) & (b / a < 2.0)), (kinds[lo // nv], a, b)
        # level 2: same launch time, split differently (conservation within timing noise)
        assert coal[2][lo:lo + nv].sum() == pytest.approx(c.sum(), rel=0.25)


def test_external_stream_join(small):
    specs, inputs = small
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        ctx = svp.Context(num_gpus=1, external_streams=[s.cuda_stream])
        vs = VPSet(ctx, specs[:10], inputs[:10], "device")
        vs.submit()
        ctx.flush()
        s.synchronize()
        for i, (sp, inp) in enumerate(zip(specs[:10], inputs[:10])):
            check_job(sp, inp, vs.output(i))
        ctx.close()


def test_residency_validation():
    ctx = svp.Context(num_gpus=1)
    va = ctx.register_kernel("vecadd")
    n = 1024
    pageable = torch.empty(n, dtype=torch.float32)
    dev = torch.empty(n, dtype=torch.float32, device="cuda")
    with pytest.raises(svp.SvpError) as e:
        ctx.submit(0, va, svp.args_vecadd(n), [(pageable.data_ptr(), 4 * n, 1, 1)] * 2 + [(dev.data_ptr(), 4 * n, 2, 0)])
    assert e.value.status == svp.SVP_E_INVAL
    with pytest.raises(svp.SvpError) as e:
        ctx.submit(0, va, svp.args_vecadd(n), [(dev.data_ptr(), 4 * n, 1, 1)] * 2 + [(dev.data_ptr(), 4 * n, 2, 0)])
    assert e.value.status == svp.SVP_E_INVAL
    ctx.close()


@pytest.mark.parametrize("level", [1, 2])
def test_residency_validation_ranges(level):
    """validate_ptrs 1 (allocation ranges remembered) and 2 (queried every submit) reject a
    buffer running past the end of its allocation, and a remembered device range declared
    HOST_PINNED; in-range buffers pass on repeated submits and compute correctly."""
    ctx = svp.Context(num_gpus=1, validate_ptrs=level)
    va = ctx.register_kernel("vecadd")
    n = 1 << 18
    a = torch.rand(n, device="cuda")
    b = torch.rand(n, device="cuda")
    c = torch.empty(n, device="cuda")
    torch.cuda.synchronize()  # filled on torch's stream; libsvp runs on its own streams
    for _ in range(2):  # the second pass hits the remembered ranges (level 1)
        ctx.submit(0, va, svp.args_vecadd(n), [(a.data_ptr(), 4 * n, 1, 0), (b.data_ptr(), 4 * n, 1, 0),
                                               (c.data_ptr(), 4 * n, 2, 0)])
        ctx.flush()
        torch.cuda.synchronize()
        assert torch.equal(c, a + b)
    big = 1 << 31  # far past any allocation holding a 1-MiB tensor
    with pytest.raises(svp.SvpError) as e:
        ctx.submit(0, va, svp.args_vecadd(big), [(a.data_ptr(), 4 * big, 1, 0), (b.data_ptr(), 4 * big, 1, 0),
                                                 (c.data_ptr(), 4 * big, 2, 0)])
    assert e.value.status == svp.SVP_E_INVAL and "past the end" in str(e.value)
    with pytest.raises(svp.SvpError) as e:
        ctx.submit(0, va, svp.args_vecadd(n), [(a.data_ptr(), 4 * n, 1, 1), (b.data_ptr(), 4 * n, 1, 0),
                                               (c.data_ptr(), 4 * n, 2, 0)])
    assert e.value.status == svp.SVP_E_INVAL
    ctx.close()


@pytest.mark.parametrize("table_mode", [0, 1])
def test_hist256_ragged_tiles_every_alignment(table_mode):
    """hist256 head/tail tiles: the producer bulk-copies their 16-B-aligned interior and
    the consumers read the < 16-B ends from global memory.  Every start offset mod 16 and
    sizes around 16 B, 32 B and the 16-KiB tile, uniform / skewed / constant data, in one
    coalesced launch; counts must equal the oracle's exactly."""
    ctx = svp.Context(num_gpus=1, table_mode=table_mode)
    kh = ctx.register_kernel("hist256")
    T = 16384
    sizes = [0, 1, 15, 16, 17, 31, 32, 33, 47, 100, T - 1, T, T + 1, T + 15, 2 * T + 7, 3 * T - 5, 5 * T + 333]
    g = np.random.default_rng(1234)
    jobs, host, bufs, counts = [], [], [], []
    vp = 0
    for off in range(16):
        for n in sizes[off % 4::4] + [sizes[(off * 7) % len(sizes)]]:
            kind = vp % 3
            if kind == 0:
                d = g.integers(0, 256, size=n, dtype=np.uint8)
            elif kind == 1:
                d = np.where(g.random(n) < 0.9, np.uint8(g.integers(0, 256)), g.integers(0, 256, size=n)).astype(np.uint8)
            else:
                d = np.full(n, 200 + off, dtype=np.uint8)
            raw = torch.empty(n + 64, dtype=torch.uint8, device="cuda")
            raw[off:off + n].copy_(torch.from_numpy(d))
            cnt = torch.full((256,), 0xDEADBEEF & 0x7FFFFFFF, dtype=torch.int32, device="cuda")
            jobs.append((vp, kh, svp.args_hist256(n), [(raw.data_ptr() + off, n, svp.DIR_IN, svp.MEM_DEVICE),
                                                      (cnt.data_ptr(), 1024, svp.DIR_OUT, svp.MEM_DEVICE)]))
            host.append(d)
            bufs.append(raw)
            counts.append(cnt)
            vp += 1
    try:
        torch.cuda.synchronize()  # buffers were filled on torch's stream; libsvp uses its own
        ctx.submit_batch(jobs)
        ctx.flush()
        torch.cuda.synchronize()
        assert ctx.flush_stats()["launches"] == 1
        for v, (d, cnt) in enumerate(zip(host, counts)):
            want = oracle.hist256(d).astype(np.int64)
            got = cnt.cpu().numpy().view(np.uint32).astype(np.int64)
            assert np.array_equal(got, want), (v, len(d))
    finally:
        ctx.close()


def test_hist256_single_launch_in_subprocess():
    """SVP_HIST_FUSED=1 (hist256 as one launch: per-launch self-resetting scratch, the last
    CTA of each VP writes its counts) is chosen once per process: run the hist parity
    tests (alignment sweep incl. empty VPs, ragged full-size cfg4, mixed small, repeated
    flushes) in a child process with the switch set."""
    import os
    import subprocess
    import sys
    here = os.path.dirname(os.path.abspath(__file__))
    cmd = [sys.executable, "-m", "pytest", os.path.join(here, "test_gpu_parity.py"), "-q", "-m", "gpu",
           "-p", "no:cacheprovider", "-k",
           "(hist256_ragged or config4 or mixed_small or repeated_flushes or config5) and not subprocess and not sgemm_full"]
    r = subprocess.run(cmd, env={**os.environ, "SVP_HIST_FUSED": "1"}, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]


def test_repeated_flushes_reuse_tables(small):
    specs, inputs = small
    ctx = svp.Context(num_gpus=1)
    vs = VPSet(ctx, specs, inputs, "device")
    uploads = []
    for r in range(3):
        vs.load_inputs()
        vs.submit()
        ctx.flush()
        uploads.append(ctx.flush_stats()["table_uploads"])
        for i, (s, inp) in enumerate(zip(specs, inputs)):
            check_job(s, inp, vs.output(i))
    assert uploads[0] == 1 and uploads[1] == 0 and uploads[2] == 0
    ctx.close()


@pytest.mark.parametrize("residency", ["device", "host"])
def test_two_logical_gpus_one_process(small, residency):
    """Single-process multi-GPU path (one issuing thread per GPU, Job Dispatcher sharding)
    on one physical B200: two logical devices mapped to CUDA ordinal 0."""
    specs, inputs = small
    ctx = svp.Context(num_gpus=2, device_ids=[0, 0], profile_level=1)
    vs = VPSet(ctx, specs, inputs, residency, device_ordinals=[0, 0])
    vs.submit()
    ctx.flush()
    ops = ctx.plan()
    devs = {op["device"] for op in ops}
    assert devs == {0, 1}
    owner = {}
    for op in ops:
        for v in op["vps"]:
            assert owner.setdefault(v, op["device"]) == op["device"]
    for i, (s, inp) in enumerate(zip(specs, inputs)):
        check_job(s, inp, vs.output(i))
    assert vs.guards_intact()
    # per-GPU Profiler view (svp_device_stats_get): every job counted once on its VP's GPU,
    # each GPU's span and kernel time measured, placement matching the plan
    ds = [ctx.device_stats(g) for g in range(2)]
    assert sum(d["jobs"] for d in ds) == len(specs)
    assert all(d["flushes"] == 1 and d["device_ns"] > 0 and d["kernel_ns"] > 0 for d in ds), ds
    assert sum(d["vps"] for d in ds) == len({s.vp for s in specs})
    for g in range(2):
        assert ds[g]["jobs"] == sum(1 for s in specs if owner.get(s.vp) == g)
    # measured timeline: every op started after the ops it waits on ended (same GPU)
    for op in ops:
        assert op["measured_start_ns"] >= 0 and op["measured_ns"] >= 0
        for w in op["waits"]:
            q = ops[w]
            if q["device"] == op["device"]:
                assert op["measured_start_ns"] + 1e3 >= q["measured_start_ns"] + q["measured_ns"], (op, q)
    ctx.reset_profile()
    assert all(ctx.device_stats(g)["jobs"] == 0 for g in range(2))
    ctx.close()


def test_ragged_grouped_sgemm_one_launch():
    """Different (M, N, K) per VP in ONE coalesced launch (FFMA and 3xTF32)."""
    dims = [(256, 512, 128), (128, 128, 512), (300, 260, 100), (64, 1024, 64), (1, 8, 8), (513, 132, 36)]
    specs = [W.JobSpec(v, "sgemm", M=M, N=N, K=K) for v, (M, N, K) in enumerate(dims)]
    inputs = inputs_for(specs)
    for impl in (svp.SGEMM_FFMA, svp.SGEMM_3XTF32):
        outs, _, st = run_svp(specs, inputs, "device", sgemm_impl=impl)
        assert st["launches"] == 1
        for s, inp, got in zip(specs, inputs, outs):
            check_job(s, inp, got)


@pytest.mark.parametrize("residency", ["device", "host"])
def test_dgemm_ragged_and_alpha_beta(residency):
    dims = [(320, 320, 320), (320, 320, 320), (65, 33, 129), (1, 1, 1), (100, 200, 0), (7, 130, 64)]
    specs = [W.JobSpec(v, "dgemm", M=M, N=N, K=K, alpha=(1.0 if v % 2 else -0.75), beta=(0.0 if v % 3 else 0.5))
             for v, (M, N, K) in enumerate(dims)]
    specs.append(W.JobSpec(9, "dgemm", M=96, N=96, K=96, int_inputs=True))
    inputs = inputs_for(specs)
    outs, _, st = run_svp(specs, inputs, residency)
    assert st["groups"] == 1
    for s, inp, got in zip(specs, inputs, outs):
        check_job(s, inp, got)


def test_table1_program_8vps():
    """The paper's Table 1 program on 8 VPs (fewer iterations): each VP multiplies two
    320x320 fp64 matrices `iters` times in program order; every level is one coalesced
    launch of 8 VPs."""
    iters = 10
    specs = W.table1_specs(nvps=8, iters=iters)
    base = [W.make_inputs(s) for s in specs[::iters]]
    inputs = [base[i // iters] for i in range(len(specs))]
    outs, _, st = run_svp(specs, inputs, "device")
    assert st["levels"] == iters and st["groups"] == iters
    want = [oracle.run_job(specs[v * iters], base[v]) for v in range(8)]
    for i, (s, got) in enumerate(zip(specs, outs)):
        check_job(s, inputs[i], got, want[i // iters])


def test_dgemm_both_tile_variants():
    """A launch with >= 2 waves of 64x64 tiles uses the 64x64 kernel, a small one the 32x32
    kernel (Table 1's 320^3 jobs); both against the oracle, ragged edges included."""
    big = [W.JobSpec(v, "dgemm", M=1000, N=1030, K=72, alpha=1.25, beta=0.5 if v == 1 else 0.0) for v in range(2)]
    big += [W.JobSpec(2 + v, "dgemm", M=640, N=640, K=40) for v in range(2)]  # 2*16*17 + 2*100 tiles
    small = [W.JobSpec(10 + v, "dgemm", M=M, N=N, K=K) for v, (M, N, K) in enumerate([(320, 320, 320), (33, 65, 17)])]
    for specs in (big, small):
        inputs = inputs_for(specs)
        outs, _, _ = run_svp(specs, inputs, "device")
        for s, inp, got in zip(specs, inputs, outs):
            check_job(s, inp, got)


def test_config5_bench_launch_config():
    """BASELINE config 5 at full size in exactly the configuration bench.py times (256 VPs,
    device-resident, interleaved, by-value segment tables, TF32+2xBF16 SGEMM on CTA pairs,
    pre-marshalled JobBatch resubmitted per step): every memory-bound VP compared in full,
    every SGEMM VP on 24 sampled elements (oracle.sgemm_element), over two consecutive
    steps (the second SAXPY step reads the first one's y; tables are reused)."""
    specs = W.config_specs(5)
    inputs = W.make_inputs_many(specs)
    stream = torch.cuda.current_stream()
    ctx = svp.Context(num_gpus=1, device_ids=[0], profile_level=1, external_streams=[stream.cuda_stream],
                      validate_ptrs=True, sgemm_impl=svp.SGEMM_TF32BF16, hetero=False, graph=False,
                      table_mode=svp.TABLE_PARAM)
    try:
        vs = VPSet(ctx, specs, inputs, "device", device_ordinals=[0])
        jobs = svp.JobBatch(vs.job_list())
        g = np.random.default_rng(5)
        prev = [dict(inp) for inp in inputs]
        for step in range(2):
            ctx.submit_batch(jobs)
            ctx.flush()
            torch.cuda.synchronize()
            st = ctx.flush_stats()
            assert st["groups"] == 5, st
            mb = [i for i, s in enumerate(specs) if s.kernel != "sgemm"]
            want = oracle.run_jobs([specs[i] for i in mb], [prev[i] for i in mb])
            outs = {}
            for i, w in zip(mb, want):
                got = vs.output(i)
                check_job(specs[i], prev[i], got, w)
                outs[i] = got
            for i, s in enumerate(specs):
                if s.kernel != "sgemm":
                    continue
                sample = [(int(g.integers(0, s.M)), int(g.integers(0, s.N))) for _ in range(20)]
                sample += [(0, 0), (s.M - 1, s.N - 1), (255, 256), (256, 255)]
                check_job(s, inputs[i], vs.output(i), sample=sample)
            for i, s in enumerate(specs):  # the next step's SAXPY reads this step's y
                if s.kernel == "saxpy":
                    prev[i] = dict(prev[i], y=outs[i]["y"].copy())
        assert vs.guards_intact()
    finally:
        ctx.close()


@pytest.mark.parametrize("impl", [svp.SGEMM_TF32BF16, svp.SGEMM_FFMA, svp.SGEMM_3XTF32])
def test_config5_sgemm_full_elementwise(impl, cfg5_sgemm_oracle):
    """the SGEMM bench.py times, at its benched shape and launch
    configuration (cfg5's 256 VPs in one interleaved flush, 51 SGEMM 2048^3 VPs in one
    coalesced launch -- wide 256 x 512 CTA-pair tiles for the default TF32+2xBF16 split;
    the FFMA and 3xTF32 implementations are the ones bench.py times beside it), compared
    ELEMENT BY ELEMENT against oracle.sgemm for the first, last and two middle SGEMM VPs
    (4 x 4.2 M outputs), on the second (steady-state) step."""
    specs, inputs, pick, want = cfg5_sgemm_oracle
    stream = torch.cuda.current_stream()
    ctx = svp.Context(num_gpus=1, device_ids=[0], profile_level=1, external_streams=[stream.cuda_stream],
                      validate_ptrs=True, sgemm_impl=impl, table_mode=svp.TABLE_PARAM)
    try:
        vs = VPSet(ctx, specs, inputs, "device", device_ordinals=[0])
        jobs = svp.JobBatch(vs.job_list())
        for _ in range(2):
            ctx.submit_batch(jobs)
            ctx.flush()
        torch.cuda.synchronize()
        st = ctx.flush_stats()
        assert st["groups"] == 5, st
        for i, w in zip(pick, want):
            got = vs.output(i)
            check_job(specs[i], inputs[i], got, w)
        assert vs.guards_intact()
    finally:
        ctx.close()


def test_dgemm_simt_kernels_in_subprocess():
    """SVP_DGEMM_DMMA=0 (read once per process): the SIMT DGEMM kernels -- 64 x 64 tiles for big
    launches, 32 x 32 ones (with split K) for small -- still meet the fp64 contract on the
    DGEMM parity cases and the Table 1 program."""
    import os
    import subprocess
    import sys
    here = os.path.dirname(os.path.abspath(__file__))
    cmd = [sys.executable, "-m", "pytest", os.path.join(here, "test_gpu_parity.py"), "-q", "-m", "gpu",
           "-p", "no:cacheprovider", "-k", "(dgemm or table1) and not subprocess"]
    r = subprocess.run(cmd, env={**os.environ, "SVP_DGEMM_DMMA": "0"}, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
