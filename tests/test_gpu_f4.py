"""GPU parity of NEXT item f4: heterogeneous coalescing (cfg hetero)
and steady-state CUDA-graph replay (cfg graph), through the C-ABI, against the oracle.

* hetero: one launch carries the vecadd / SAXPY / Black-Scholes segments of a level; every
  output must equal the oracle AND be bit-identical to the homogeneous launches (same tile
  bodies, same per-element instruction sequence).
* graph: flush 1 plans and runs directly, flush 2 (same requests) reuses the plan and
  captures a graph, flush 3+ replay it.  The replayed work must read the buffers' CURRENT
  contents (new inputs every flush) and the profiler must still attribute every op."""
import numpy as np
import pytest
import torch

import workloads as W
from gpu_common import check_job, inputs_for, run_svp
from paper_conf_dac_jungc15_b200 import svp
from paper_conf_dac_jungc15_b200.vpset import VPSet

pytestmark = pytest.mark.gpu


def _bits(a):
    return a.view(np.uint32) if a.dtype == np.float32 else a


@pytest.fixture(scope="module")
def small():
    specs = W.mixed_small(nvps=40, max_n=90000)
    return specs, inputs_for(specs)


@pytest.mark.parametrize("residency", ["device", "host"])
def test_hetero_parity_and_bit_identity(small, residency):
    specs, inputs = small
    a, _, st = run_svp(specs, inputs, residency, hetero=True)
    b, _, _ = run_svp(specs, inputs, residency, hetero=False)
    for s, inp, x, y in zip(specs, inputs, a, b):
        check_job(s, inp, x)
        for k in x:
            assert np.array_equal(_bits(x[k]), _bits(y[k])), (s.vp, s.kernel, k)
    if residency == "device":
        assert st["groups"] == 3  # ew-mix + hist256 + sgemm


def test_hetero_config4_full_size():
    """cfg4 sizes (ragged 64Ki-16Mi, adversarial sizes, misaligned views) in one mixed launch."""
    specs = [s for s in W.config_specs(4) if s.kernel in ("vecadd", "saxpy", "blackscholes")]
    inputs = W.make_inputs_many(specs)
    outs, _, st = run_svp(specs, inputs, "device", hetero=True, profile_level=1)
    assert st["launches"] == 1
    for s, inp, got in zip(specs, inputs, outs):
        check_job(s, inp, got)


@pytest.mark.parametrize("residency", ["device", "host"])
@pytest.mark.parametrize("hetero", [False, True])
def test_graph_replay_reads_fresh_inputs(small, residency, hetero):
    specs, _ = small
    ctx = svp.Context(num_gpus=1, graph=True, hetero=hetero, profile_level=1)
    try:
        vs = VPSet(ctx, specs, None, residency)
        jb = svp.JobBatch(vs.job_list())
        seen = []
        for r in range(4):
            inputs = inputs_for(specs, seed=W.BASE_SEED + 17 * r)
            vs.inputs = inputs
            vs.load_inputs()
            ctx.submit_batch(jb)
            ctx.flush()
            torch.cuda.synchronize()
            st = ctx.flush_stats()
            seen.append((st["plan_reused"], st["graph_replays"]))
            for i, (s, inp) in enumerate(zip(specs, inputs)):
                check_job(s, inp, vs.output(i))
            ops = ctx.plan()
            assert all(op["measured_ns"] >= 0 for op in ops), r
            per = [ctx.profile(s.vp) for s in specs]
        assert seen == [(0, 0), (1, 1), (1, 1), (1, 1)]
        assert vs.guards_intact()
        k_tot = ctx.profile(-1)["kernel_ns"]
        assert sum(p["kernel_ns"] for p in per) == pytest.approx(k_tot, rel=1e-9)
    finally:
        ctx.close()


def test_graph_replans_when_requests_change(small):
    specs, inputs = small
    ctx = svp.Context(num_gpus=1, graph=True)
    try:
        vs = VPSet(ctx, specs, inputs, "device")
        for r in range(3):
            vs.load_inputs()
            vs.submit()
            ctx.flush()
        assert ctx.flush_stats()["graph_replays"] == 1
        # a different request set (first 10 VPs only): new plan, direct issue, correct
        sub = VPSet(ctx, specs[:10], inputs[:10], "device")
        sub.submit()
        ctx.flush()
        st = ctx.flush_stats()
        assert st["plan_reused"] == 0 and st["graph_replays"] == 0
        torch.cuda.synchronize()
        for i, (s, inp) in enumerate(zip(specs[:10], inputs[:10])):
            check_job(s, inp, sub.output(i))
    finally:
        ctx.close()


@pytest.mark.parametrize("table_mode", [svp.TABLE_GLOBAL, svp.TABLE_PARAM])
def test_graph_alternating_buffer_sets(small, table_mode):
    """A serving loop that rotates input buffer sets (ping-pong, or bench.py's sets that keep
    the working set out of L2) alternates between plans.  Each set's plan is cached and its
    graph replayed with that plan's OWN copy of the device tables (segment tables, SGEMM
    tensor maps): a replay must never read the tables another set's flush uploaded.  Fresh
    inputs every round, every output against the oracle."""
    specs, _ = small
    ctx = svp.Context(num_gpus=1, graph=True, profile_level=1, table_mode=table_mode)
    try:
        sets = [VPSet(ctx, specs, None, "device") for _ in range(3)]
        jbs = [svp.JobBatch(vs.job_list()) for vs in sets]
        seen = []
        for r in range(9):
            k = r % 3
            inputs = inputs_for(specs, seed=W.BASE_SEED + 31 * r)
            sets[k].inputs = inputs
            sets[k].load_inputs()
            ctx.submit_batch(jbs[k])
            ctx.flush()
            torch.cuda.synchronize()
            st = ctx.flush_stats()
            seen.append((st["plan_reused"], st["graph_replays"]))
            for i, (s, inp) in enumerate(zip(specs, inputs)):
                check_job(s, inp, sets[k].output(i))
        # round 0-2: three fresh plans; 3-5: second sightings (reused plan, captured graph
        # replayed once); 6-8: replays
        assert seen == [(0, 0)] * 3 + [(1, 1)] * 6, seen
        assert all(vs.guards_intact() for vs in sets)
    finally:
        ctx.close()


def test_serial_graph_baseline_b3(small):
    """B3: the serial per-job launches captured in a graph are still
    per-VP correct."""
    specs, inputs = small
    ctx = svp.Context(num_gpus=1, graph=True, coalesce=False, interleave=False)
    try:
        vs = VPSet(ctx, specs, inputs, "device")
        for r in range(3):
            vs.load_inputs()
            vs.submit()
            ctx.flush()
        st = ctx.flush_stats()
        assert st["graph_replays"] == 1 and st["launches"] == len(specs)
        torch.cuda.synchronize()
        for i, (s, inp) in enumerate(zip(specs, inputs)):
            check_job(s, inp, vs.output(i))
    finally:
        ctx.close()


@pytest.mark.parametrize("residency", ["device", "host"])
@pytest.mark.parametrize("hetero", [False, True])
def test_table_mode_param(small, residency, hetero):
    """SURVEY §8(b) table_mode: segment tables passed by value (kernel parameter) give the
    same bits as the global table; GEMM launches keep the global table."""
    specs, inputs = small
    a, _, sa = run_svp(specs, inputs, residency, table_mode=svp.TABLE_PARAM, hetero=hetero)
    b, _, _ = run_svp(specs, inputs, residency, table_mode=svp.TABLE_GLOBAL, hetero=hetero)
    for s, inp, x, y in zip(specs, inputs, a, b):
        check_job(s, inp, x)
        for k in x:
            assert np.array_equal(_bits(x[k]), _bits(y[k])), (s.vp, s.kernel, k)


def test_table_mode_param_no_upload_and_fallback():
    """Elementwise-only flushes in param mode upload no table (groups of 16 and of 17..64
    VPs use the 1-KiB and 4-KiB parameter blocks); a group larger than the parameter table
    (64 VPs) falls back to the global table and stays correct."""
    few = [W.JobSpec(v, ("vecadd", "saxpy", "hist256", "blackscholes")[v % 4], n=5000 + 77 * v) for v in range(40)]
    cap16 = [W.JobSpec(v, ("hist256", "saxpy")[v % 2], n=3000 + 91 * v) for v in range(32)]
    cap64 = [W.JobSpec(v, ("vecadd", "hist256")[v % 2], n=2000 + 51 * v) for v in range(128)]
    over = [W.JobSpec(v, "hist256", n=1000 + 29 * v) for v in range(65)]
    many = [W.JobSpec(v, "vecadd", n=1000 + 13 * v) for v in range(300)]
    for specs, uploads in ((few, 0), (cap16, 0), (cap64, 0), (over, 1), (many, 1)):
        inputs = inputs_for(specs)
        outs, _, st = run_svp(specs, inputs, "device", table_mode=svp.TABLE_PARAM)
        assert st["table_uploads"] == uploads
        for s, inp, got in zip(specs, inputs, outs):
            check_job(s, inp, got)


def test_table_mode_param_with_graph(small):
    specs, _ = small
    ctx = svp.Context(num_gpus=1, graph=True, table_mode=svp.TABLE_PARAM)
    try:
        vs = VPSet(ctx, specs, None, "device")
        jb = svp.JobBatch(vs.job_list())
        for r in range(3):
            inputs = inputs_for(specs, seed=W.BASE_SEED + 5 * r)
            vs.inputs = inputs
            vs.load_inputs()
            ctx.submit_batch(jb)
            ctx.flush()
            torch.cuda.synchronize()
            for i, (s, inp) in enumerate(zip(specs, inputs)):
                check_job(s, inp, vs.output(i))
        assert ctx.flush_stats()["graph_replays"] == 1
    finally:
        ctx.close()
