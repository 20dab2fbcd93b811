"""Failure handling on the GPU (run in subprocesses: a faulting kernel poisons the CUDA
context of its process): a device fault makes svp_flush return SVP_E_CUDA and the context
sticky-errored (SVP_E_STATE afterwards, svp_wait of its jobs fails), and the flush
watchdog reports SVP_E_TIMEOUT."""
import subprocess
import sys
import textwrap

import pytest

pytestmark = pytest.mark.gpu


def _run(code):
    r = subprocess.run([sys.executable, "-c", textwrap.dedent(code)], capture_output=True, text=True, timeout=300)
    return r.returncode, r.stdout + r.stderr


def test_device_fault_is_sticky():
    rc, out = _run("""
        import sys; sys.path.insert(0, '.')
        import torch
        from paper_conf_dac_jungc15_b200 import svp
        ctx = svp.Context(num_gpus=1, validate_ptrs=False)
        k = ctx.register_kernel('vecadd')
        n = 1 << 20
        good = torch.ones(n, device='cuda')
        bad = 0x10  # unmapped device address
        j = ctx.submit(0, k, svp.args_vecadd(n), [(bad, 4 * n, 1, 0), (good.data_ptr(), 4 * n, 1, 0), (good.data_ptr(), 4 * n, 2, 0)])
        try:
            ctx.flush(); print('NO_ERROR')
        except svp.SvpError as e:
            print('FLUSH', e.status)
        try:
            ctx.submit(1, k, svp.args_vecadd(0), [(0, 0, 1, 0)] * 2 + [(0, 0, 2, 0)]); print('SUBMIT_OK')
        except svp.SvpError as e:
            print('SUBMIT', e.status)
        try:
            ctx.wait(j, 1000); print('WAIT_OK')
        except svp.SvpError as e:
            print('WAIT', e.status)
        ctx.close(); print('CLOSED')
    """)
    assert "FLUSH -3" in out, out          # SVP_E_CUDA
    assert "SUBMIT -5" in out, out         # SVP_E_STATE afterwards
    assert "WAIT -3" in out, out           # the job's flush failed
    assert "CLOSED" in out, out


def test_flush_watchdog_timeout():
    rc, out = _run("""
        import sys; sys.path.insert(0, '.')
        import torch
        from paper_conf_dac_jungc15_b200 import svp
        ctx = svp.Context(num_gpus=1, flush_timeout_ms=1, sgemm_impl=svp.SGEMM_FFMA)
        k = ctx.register_kernel('sgemm')
        n = 8192
        A = torch.rand(n, n, device='cuda'); B = torch.rand(n, n, device='cuda'); C = torch.empty(n, n, device='cuda')
        torch.cuda.synchronize()
        ctx.submit(0, k, svp.args_sgemm(n, n, n), [(A.data_ptr(), 4 * n * n, 1, 0), (B.data_ptr(), 4 * n * n, 1, 0), (C.data_ptr(), 4 * n * n, 2, 0)])
        try:
            ctx.flush(); print('NO_TIMEOUT')
        except svp.SvpError as e:
            print('FLUSH', e.status)
        ctx.close(); print('CLOSED')
    """)
    assert "FLUSH -6" in out, out          # SVP_E_TIMEOUT
    assert "CLOSED" in out, out
