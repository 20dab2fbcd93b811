"""Cross-process IPC front end (the paper's IPC Manager) on CPU.

A server process owns a dry-run context (no CUDA); separate VP *processes* connect to
the shared-memory segment, allocate arena buffers, submit jobs through the ticket ring
and wait for them.  Checks the protocol: every ticket completes exactly once, bad
requests fail per job, jobs of many processes coalesce, a vanished server is reported."""
import multiprocessing as mp
import os
import uuid

import pytest

from paper_conf_dac_jungc15_b200 import svp


def _client(name, vp0, nvps, calls, q):
    try:
        from paper_conf_dac_jungc15_b200 import svp as s
        c = s.IpcClient(name)
        k = s.kernel_lookup("vecadd")
        n = 1000
        bufs = []
        for v in range(nvps):
            offs = [c.alloc(4 * n)[0] for _ in range(3)]
            bufs.append([(offs[0], 4 * n, s.DIR_IN), (offs[1], 4 * n, s.DIR_IN), (offs[2], 4 * n, s.DIR_OUT)])
        done = 0
        for _ in range(calls):
            tickets = [c.submit(vp0 + v, k, s.args_vecadd(n), bufs[v]) for v in range(nvps)]
            for t in tickets:
                c.wait(t, timeout_ms=20000)
                done += 1
        c.close()
        q.put(("ok", done))
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put(("err", repr(e)))


def _name():
    return "svp_test_" + uuid.uuid4().hex[:12]


def test_ipc_many_processes_dry_run():
    name = _name()
    ctx = svp.Context(dry_run=True)
    ctx.register_kernel("vecadd")
    with svp.IpcServer(ctx, name, arena_bytes=16 << 20, nslots=64) as srv:
        mpx = mp.get_context("spawn")
        q = mpx.Queue()
        procs = [mpx.Process(target=_client, args=(name, 100 * p, 4, 10, q)) for p in range(3)]
        for p in procs:
            p.start()
        res = [q.get(timeout=120) for _ in procs]
        for p in procs:
            p.join(60)
        assert all(r[0] == "ok" for r in res), res
        assert sum(r[1] for r in res) == 3 * 4 * 10
        st = srv.stats()
        assert st["served"] == 120 and st["tickets"] == 120
    ctx.close()
    assert not os.path.exists("/dev/shm/" + name)


def test_ipc_bad_request_fails_that_job_only():
    name = _name()
    ctx = svp.Context(dry_run=True)
    ctx.register_kernel("vecadd")
    with svp.IpcServer(ctx, name, arena_bytes=1 << 20, nslots=8):
        c = svp.IpcClient(name)
        k = svp.kernel_lookup("vecadd")
        off = c.alloc(4096)[0]
        bad = c.submit(0, k, svp.args_vecadd(1000), [(off, 4000, 1), (1 << 40, 4000, 1), (off, 4000, 2)])
        with pytest.raises(svp.SvpError) as e:
            c.wait(bad, timeout_ms=10000)
        assert e.value.status == svp.SVP_E_INVAL
        good = c.submit(0, k, svp.args_vecadd(100), [(off, 400, 1), (off + 1024, 400, 1), (off + 2048, 400, 2)])
        c.wait(good, timeout_ms=10000)
        with pytest.raises(svp.SvpError):
            c.wait(good, timeout_ms=10)  # a ticket is waited once
        c.close()
    ctx.close()


def test_ipc_server_gone_and_errors():
    with pytest.raises(svp.SvpError):
        svp.IpcClient(_name())  # no such segment
    name = _name()
    ctx = svp.Context(dry_run=True)
    srv = svp.IpcServer(ctx, name, arena_bytes=1 << 20, nslots=4)
    c = svp.IpcClient(name)
    with pytest.raises(svp.SvpError) as e:
        c.alloc(2 << 20)
    assert e.value.status == svp.SVP_E_NOMEM
    srv.shutdown()
    with pytest.raises(svp.SvpError) as e:
        c.submit(0, 1, svp.args_vecadd(0), [])
    assert e.value.status == svp.SVP_E_STATE
    c.close()
    ctx.close()
    assert svp.kernel_lookup("sgemm") == 5
