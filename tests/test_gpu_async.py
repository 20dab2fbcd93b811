"""Pipelined flushes (svp_flush_async / svp_flush_wait, ABI 6) against the oracle.

A flush stays pending until the next flush has been issued.  So while flush i's kernels
run, the host plans and issues flush i+1.  These tests check four things:
* every flush's outputs equal the oracle once it has completed;
* completion happens when the API says: at the next flush, at svp_flush_wait, at svp_wait
  on one of its jobs;
* svp_flush_stats reports the last completed flush;
* rotating buffer sets, host-resident staging, graph replay, profiling (no overlap) and two
  logical GPUs all stay correct."""
import pytest
import torch

import workloads as W
from gpu_common import check_job, inputs_for
from paper_conf_dac_jungc15_b200 import svp
from paper_conf_dac_jungc15_b200.vpset import VPSet

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def specs():
    return W.mixed_small(nvps=24, max_n=60000)


def _pipeline(ctx, specs, residency, rounds=7, nsets=3, device_ordinals=None):
    """Round r refreshes set r % nsets with new inputs (that set's previous flush, r - nsets,
    has completed), submits it and flushes async.  On return, flush r - 1 has completed and
    is checked; the last one is completed by flush_wait."""
    sets = [VPSet(ctx, specs, None, residency, device_ordinals=device_ordinals) for _ in range(nsets)]
    jbs = [svp.JobBatch(vs.job_list()) for vs in sets]
    expect = {}
    tickets = []
    for r in range(rounds):
        k = r % nsets
        inputs = inputs_for(specs, seed=W.BASE_SEED + 101 * r)
        sets[k].inputs = inputs
        sets[k].load_inputs()
        ctx.submit_batch(jbs[k])
        tickets.append(ctx.flush_async())
        expect[r] = (k, inputs)
        if r >= 1:
            # flush r - 1 completed when flush r was issued
            assert ctx.flush_stats()["jobs"] == len(specs)
            kp, inp_prev = expect.pop(r - 1)
            torch.cuda.synchronize()
            for i, (s, inp) in enumerate(zip(specs, inp_prev)):
                check_job(s, inp, sets[kp].output(i))
    ctx.flush_wait(tickets[-1])
    k, inp_last = expect.pop(rounds - 1)
    torch.cuda.synchronize()
    for i, (s, inp) in enumerate(zip(specs, inp_last)):
        check_job(s, inp, sets[k].output(i))
    assert tickets == list(range(tickets[0], tickets[0] + rounds))
    assert all(vs.guards_intact() for vs in sets)


@pytest.mark.parametrize("residency", ["device", "host"])
@pytest.mark.parametrize("graph", [True, False])
def test_async_pipeline_parity(specs, residency, graph):
    ctx = svp.Context(num_gpus=1, graph=graph)
    try:
        _pipeline(ctx, specs, residency)
    finally:
        ctx.close()


def test_async_with_profiling_completes_in_order(specs):
    """profile_level 1: no overlap (the previous flush completes before the next issues),
    results and per-op timings still right."""
    ctx = svp.Context(num_gpus=1, profile_level=1)
    try:
        _pipeline(ctx, specs, "device", rounds=4)
        assert all(op["measured_ns"] >= 0 for op in ctx.plan())
    finally:
        ctx.close()


def test_async_two_logical_gpus(specs):
    ctx = svp.Context(num_gpus=2, device_ids=[0, 0])
    try:
        _pipeline(ctx, specs, "device", rounds=5, device_ordinals=[0, 0])
    finally:
        ctx.close()


def test_svp_wait_completes_a_pending_flush(specs):
    """VP Control on a job of the pending async flush: svp_wait completes that flush itself."""
    inputs = inputs_for(specs)
    ctx = svp.Context(num_gpus=1)
    try:
        vs = VPSet(ctx, specs, inputs, "device")
        ids = vs.submit()
        ctx.flush_async()
        ctx.wait(ids[-1])
        for i, (s, inp) in enumerate(zip(specs, inputs)):
            check_job(s, inp, vs.output(i))
        # then a synchronous flush of a second set: both results stand
        inputs2 = inputs_for(specs, seed=W.BASE_SEED + 5)
        vs2 = VPSet(ctx, specs, inputs2, "device")
        vs2.submit()
        ctx.flush()
        for i, (s, inp) in enumerate(zip(specs, inputs2)):
            check_job(s, inp, vs2.output(i))
    finally:
        ctx.close()


def test_async_stats_report_last_completed(specs):
    """Flushes of different sizes: after flush_async of flush r, the stats are flush r - 1's."""
    inputs = inputs_for(specs)
    ctx = svp.Context(num_gpus=1)
    try:
        vs = VPSet(ctx, specs, inputs, "device")
        jl = vs.job_list()
        # disjoint VP slices (saxpy's y is in-out: each VP runs exactly once)
        cuts = [0, 3, 8, 15, 24]
        sizes = [b - a for a, b in zip(cuts, cuts[1:])]
        for r, n in enumerate(sizes):
            ctx.submit_batch(jl[cuts[r]:cuts[r + 1]])
            t = ctx.flush_async()
            if r:
                assert ctx.flush_stats()["jobs"] == sizes[r - 1]
        ctx.flush_wait(t)
        assert ctx.flush_stats()["jobs"] == sizes[-1]
        for i, (s, inp) in enumerate(zip(specs, inputs)):
            check_job(s, inp, vs.output(i))
    finally:
        ctx.close()


def test_finalize_completes_a_pending_flush(specs):
    inputs = inputs_for(specs)
    ctx = svp.Context(num_gpus=1)
    vs = VPSet(ctx, specs, inputs, "device")
    vs.submit()
    ctx.flush_async()
    ctx.close()  # waits for the pending flush before tearing down
    torch.cuda.synchronize()
    for i, (s, inp) in enumerate(zip(specs, inputs)):
        check_job(s, inp, vs.output(i))
