"""VP Control on the GPU: VP threads issue synchronous SAXPY calls (submit + svp_wait)
served by the continuous dispatcher; every VP's result equals the oracle's sequential
program (bit-exact), and concurrent VPs' calls coalesce into shared launches."""
import threading

import numpy as np
import pytest
import torch

import oracle
import workloads as W
from paper_conf_dac_jungc15_b200 import svp

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("window_us", [0, 100])
def test_sync_vps_through_dispatcher(window_us):
    nvps, calls, n = 16, 20, 50001
    ctx = svp.Context(num_gpus=1)
    k = ctx.register_kernel("saxpy")
    xs, ys, want = [], [], []
    for v in range(nvps):
        g = W.rng(21, v, 1)
        x, y = W.uniform_f32(g, n, -1, 1), W.uniform_f32(g, n, -1, 1)
        a = 0.25 + 0.01 * v
        yy = y.copy()
        for _ in range(calls):
            yy = oracle.saxpy(a, x, yy)
        want.append(yy)
        xs.append(torch.from_numpy(x).cuda())
        ys.append(torch.from_numpy(y).cuda())
    torch.cuda.synchronize()
    ctx.start_dispatcher(window_us=window_us)
    errors = []

    def program(v):
        try:
            a = 0.25 + 0.01 * v
            bufs = [(xs[v].data_ptr(), 4 * n, svp.DIR_IN, svp.MEM_DEVICE),
                    (ys[v].data_ptr(), 4 * n, svp.DIR_INOUT, svp.MEM_DEVICE)]
            for _ in range(calls):
                j = ctx.submit(v, k, svp.args_saxpy(n, a), bufs)
                ctx.wait(j, timeout_ms=60000)
        except Exception as e:  # pragma: no cover
            errors.append(e)

    ts = [threading.Thread(target=program, args=(v,)) for v in range(nvps)]
    for t in ts:
        t.start()
    for t in ts:
        t.join(120)
    ctx.stop_dispatcher()
    assert not errors
    prof = ctx.profile(-1)
    assert prof["jobs"] == nvps * calls
    # coalescing happened: fewer launches than jobs
    assert prof["launches"] < nvps * calls
    for v in range(nvps):
        assert np.array_equal(ys[v].cpu().numpy(), want[v]), v
    ctx.close()
