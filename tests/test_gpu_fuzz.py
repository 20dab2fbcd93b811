"""Randomised flush sequences against the oracle (GPU).

Each round submits two VP sets, one device-resident and one host-resident (pinned, staged
through the arena), and flushes them with svp_flush_async. The sets have random kernels
(vecadd, SAXPY, hist256, Black-Scholes, SGEMM), ragged sizes (0, 1, unaligned, several
tiles), misaligned views and random SGEMM alpha/beta. Some VPs submit a second job in the same
flush, which gives a second level that must run after the first in program order.

The arena is a few MiB, so host-resident chunks wrap it, and the ring's ordering
 is exercised on the device with mixed residency. Round r is checked once
round r+1 has been issued, because issuing r+1 completes r. That includes the in-out
SAXPY y and the two-level VPs.
"""
import dataclasses

import numpy as np
import pytest
import torch

import oracle
import workloads as W
from gpu_common import check_job, inputs_for
from paper_conf_dac_jungc15_b200 import svp
from paper_conf_dac_jungc15_b200.vpset import VPSet

pytestmark = pytest.mark.gpu

KERNELS = ("vecadd", "saxpy", "hist256", "blackscholes", "sgemm")


def _random_specs(rng, vp0, nvps):
    specs = []
    for i in range(nvps):
        vp = vp0 + i
        k = KERNELS[int(rng.integers(0, len(KERNELS)))]
        if k == "sgemm":
            M, N, K = (int(x) for x in rng.integers(1, 300, size=3))
            N = max(4, N // 4 * 4)
            K = max(4, K // 4 * 4)
            beta = float(rng.choice([0.0, 0.0, 0.5]))
            s = W.JobSpec(vp, k, M=M, N=N, K=K, alpha=float(rng.choice([1.0, -1.5])), beta=beta)
        else:
            n = int(rng.choice([0, 1, 5, 4095, 4097, int(rng.integers(1, 200000))]))
            s = W.JobSpec(vp, k, n=n, misalign=int(rng.integers(0, 2)), skew=bool(k == "hist256" and rng.integers(0, 2)))
        W._scalar_for(W.BASE_SEED + vp, s)
        specs.append(s)
    return specs


def _expected(specs, inputs):
    """Per spec (in submission order) the oracle's outputs; a VP's second job runs on the
    first job's outputs where they share a buffer (not the case here: every spec owns its
    buffers), so each job is checked on its own inputs."""
    return oracle.run_jobs(specs, inputs)


@pytest.mark.parametrize("seed", [11, 12, 13, 14, 15])
def test_async_fuzz_mixed_residency(seed):
    rng = np.random.default_rng(seed)
    ctx = svp.Context(num_gpus=1, arena_bytes=6 << 20)
    pending = None
    try:
        for r in range(8):
            vp0 = 1000 * (r + 1)
            dev_specs = _random_specs(rng, vp0, int(rng.integers(3, 14)))
            host_specs = _random_specs(rng, vp0 + 500, int(rng.integers(3, 14)))
            # a second job of some device VPs in the same flush (level 1, program order)
            dev_specs += [dataclasses.replace(s) for s in dev_specs[: int(rng.integers(0, 3))]]
            dev_inputs = inputs_for(dev_specs, seed=W.BASE_SEED + 7 * r + seed)
            host_inputs = inputs_for(host_specs, seed=W.BASE_SEED + 7 * r + seed + 3)
            dev = VPSet(ctx, dev_specs, dev_inputs, "device")
            host = VPSet(ctx, host_specs, host_inputs, "host")
            torch.cuda.synchronize()
            dev.submit()
            host.submit()
            ticket = ctx.flush_async()
            if pending is not None:
                _check(*pending)
            pending = (dev, dev_specs, dev_inputs, host, host_specs, host_inputs)
        ctx.flush_wait(ticket)  # completes the last async flush
        _check(*pending)
        st = ctx.flush_stats()
        assert st["jobs"] > 0
    finally:
        ctx.close()


def _check(dev, dev_specs, dev_inputs, host, host_specs, host_inputs):
    torch.cuda.synchronize()
    for vs, specs, inputs in ((dev, dev_specs, dev_inputs), (host, host_specs, host_inputs)):
        want = _expected(specs, inputs)
        for i, (s, inp, w) in enumerate(zip(specs, inputs, want)):
            check_job(s, inp, vs.output(i), w)
        assert vs.guards_intact()
