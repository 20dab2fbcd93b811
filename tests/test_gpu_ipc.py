"""IPC front end on the GPU: VP processes (no CUDA in them) run SAXPY programs on buffers
in the shared arena through a server process's svp context; results are bit-exact with
the oracle's sequential program."""
import multiprocessing as mp
import uuid

import numpy as np
import pytest

pytestmark = pytest.mark.gpu


def _vp_process(name, vps, calls, n, q):
    try:
        import ctypes
        import oracle
        import workloads as W
        from paper_conf_dac_jungc15_b200 import svp
        c = svp.IpcClient(name)
        k = svp.kernel_lookup("saxpy")
        views, bufs, want = [], [], []
        for v in vps:
            (ox, px), (oy, py) = c.alloc(4 * n), c.alloc(4 * n)
            x = np.ctypeslib.as_array((ctypes.c_float * n).from_address(px))
            y = np.ctypeslib.as_array((ctypes.c_float * n).from_address(py))
            g = W.rng(33, v, 1)
            x[:] = W.uniform_f32(g, n, -1, 1)
            y[:] = W.uniform_f32(g, n, -1, 1)
            a = 0.5 + 0.01 * v
            yy = y.copy()
            for _ in range(calls):
                yy = oracle.saxpy(a, x.copy(), yy)
            want.append(yy)
            views.append(y)
            bufs.append([(ox, 4 * n, svp.DIR_IN), (oy, 4 * n, svp.DIR_INOUT)])
        for _ in range(calls):
            ts = [c.submit(v, k, svp.args_saxpy(n, 0.5 + 0.01 * v), bufs[i]) for i, v in enumerate(vps)]
            for t in ts:
                c.wait(t, timeout_ms=60000)
        ok = all(np.array_equal(views[i], want[i]) for i in range(len(vps)))
        c.close()
        q.put(("ok", ok))
    except Exception as e:  # pragma: no cover
        q.put(("err", repr(e)))


def test_ipc_vp_processes_saxpy():
    from paper_conf_dac_jungc15_b200 import svp
    name = "svp_gpu_" + uuid.uuid4().hex[:10]
    ctx = svp.Context(num_gpus=1, profile_level=1)
    ctx.register_kernel("saxpy")
    with svp.IpcServer(ctx, name, arena_bytes=256 << 20, nslots=256) as srv:
        mpx = mp.get_context("spawn")
        q = mpx.Queue()
        procs = [mpx.Process(target=_vp_process, args=(name, list(range(4 * p, 4 * p + 4)), 8, 100003, q))
                 for p in range(3)]
        for p in procs:
            p.start()
        res = [q.get(timeout=300) for _ in procs]
        for p in procs:
            p.join(60)
        assert res == [("ok", True)] * 3, res
        assert srv.stats()["served"] == 3 * 4 * 8
    prof = ctx.profile(-1)
    assert prof["jobs"] == 96 and prof["launches"] < 96  # coalesced across VP processes
    assert prof["bytes_h2d"] > 0 and prof["bytes_d2h"] > 0
    ctx.close()
