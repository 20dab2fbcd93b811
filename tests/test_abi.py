"""libsvp C-ABI: the library loads, exports every symbol include/svp.h declares, and
rejects bad requests with the documented status codes (CPU only: dry-run contexts)."""
import os
import re

import pytest
import torch

from paper_conf_dac_jungc15_b200 import svp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _header_functions():
    src = open(os.path.join(ROOT, "include", "svp.h")).read()
    decl = r"^\s*(?:svp_status|void|const char\s*\*|int32_t)\s*(svp_[a-z_]+)\s*\("
    return sorted(set(re.findall(decl, src, flags=re.M)))


def test_library_exports_every_declared_symbol():
    L = svp.load()
    declared = _header_functions()
    assert set(declared) == set(svp.EXPORTS), (set(declared) ^ set(svp.EXPORTS))
    for name in declared:
        assert hasattr(L, name), name
    assert L.svp_abi_version() == 6


@pytest.mark.skipif(bool(os.environ.get("SVP_LIB")), reason="SVP_LIB selects a sanitizer build on purpose")
def test_lib_is_the_in_tree_build():
    L = svp.load()
    assert os.path.dirname(os.path.abspath(L._name)) == os.path.join(ROOT, "paper_conf_dac_jungc15_b200")


def test_config_default():
    cfg = svp.svp_config()
    svp.load().svp_config_default(cfg)
    assert cfg.streams_per_gpu == 4 and cfg.coalesce == 1 and cfg.interleave == 1 and cfg.max_chunks == 8
    assert cfg.validate_ptrs == 1 and cfg.dry_run == 0 and cfg.sgemm_impl == svp.SGEMM_TF32BF16
    assert cfg.table_mode == svp.TABLE_PARAM and cfg.hetero == 0 and cfg.graph == 1 and cfg.sgemm_kchunk == 768


@pytest.mark.skipif(torch.cuda.is_available(), reason="needs a host without GPUs")
def test_init_without_gpu_fails_loudly():
    with pytest.raises(svp.SvpError) as e:
        svp.Context()
    assert e.value.status == svp.SVP_E_CUDA


@pytest.mark.parametrize("kw", [dict(streams_per_gpu=0), dict(validate_ptrs=3), dict(validate_ptrs=-1),
                                dict(table_mode=2), dict(profile_level=3)])
def test_init_rejects_bad_config(kw):
    with pytest.raises(svp.SvpError) as e:
        svp.Context(dry_run=True, **kw)
    assert e.value.status == svp.SVP_E_INVAL


def test_register_kernels():
    with svp.Context(dry_run=True) as c:
        ids = [c.register_kernel(k) for k in ("vecadd", "saxpy", "hist256", "blackscholes", "sgemm")]
        assert len(set(ids)) == 5
        assert c.register_kernel("vecadd") == ids[0]  # idempotent
        with pytest.raises(svp.SvpError) as e:
            c.register_kernel("conv2d")
        assert e.value.status == svp.SVP_E_NOKERNEL


FAKE = 0x7F0000000000  # dry-run contexts never touch buffers


def _vecadd_bufs(n, mem=svp.MEM_DEVICE, bytes_=None):
    b = 4 * n if bytes_ is None else bytes_
    return [(FAKE, b, svp.DIR_IN, mem), (FAKE + 2**30, b, svp.DIR_IN, mem), (FAKE + 2**31, b, svp.DIR_OUT, mem)]


@pytest.mark.parametrize("case,status", [
    ("wrong_nbufs", svp.SVP_E_INVAL), ("wrong_dir", svp.SVP_E_INVAL), ("too_small", svp.SVP_E_INVAL),
    ("bad_vp", svp.SVP_E_INVAL), ("unregistered", svp.SVP_E_NOKERNEL), ("short_args", svp.SVP_E_INVAL),
    ("null_ptr", svp.SVP_E_INVAL), ("bad_mem", svp.SVP_E_INVAL), ("sgemm_beta_out", svp.SVP_E_INVAL),
])
def test_submit_validation(case, status):
    with svp.Context(dry_run=True) as c:
        va = c.register_kernel("vecadd")
        sg = c.register_kernel("sgemm")
        n = 1000
        vp, kid, args, bufs = 0, va, svp.args_vecadd(n), _vecadd_bufs(n)
        if case == "wrong_nbufs":
            bufs = bufs[:2]
        elif case == "wrong_dir":
            bufs[2] = (bufs[2][0], bufs[2][1], svp.DIR_IN, svp.MEM_DEVICE)
        elif case == "too_small":
            bufs = _vecadd_bufs(n, bytes_=4 * n - 4)
        elif case == "bad_vp":
            vp = 1 << 20
        elif case == "unregistered":
            kid = 3
        elif case == "short_args":
            args = b"\x01\x00"
        elif case == "null_ptr":
            bufs[0] = (0, 4 * n, svp.DIR_IN, svp.MEM_DEVICE)
        elif case == "bad_mem":
            bufs[1] = (bufs[1][0], bufs[1][1], svp.DIR_IN, 7)
        elif case.startswith("sgemm"):
            kid = sg
            M, N, K = 64, 64, 64
            beta = 0.0
            dirc = svp.DIR_OUT
            base = FAKE
            if case == "sgemm_k":
                K = 30
            if case == "sgemm_beta_out":
                beta = 1.0
            if case == "sgemm_misaligned":
                base = FAKE + 4
            args = svp.args_sgemm(M, N, K, 1.0, beta)
            bufs = [(base, 4 * M * K, svp.DIR_IN, 0), (FAKE + 2**30, 4 * K * N, svp.DIR_IN, 0),
                    (FAKE + 2**31, 4 * M * N, dirc, 0)]
        with pytest.raises(svp.SvpError) as e:
            c.submit(vp, kid, args, bufs)
        assert e.value.status == status, svp.last_error()
        assert svp.last_error()


def test_sgemm_any_shape_and_alignment_is_accepted_and_routed():
    """K or N not a multiple of 4 (a TMA row pitch must be a multiple
    of 16 B) and device buffers not 16-B aligned used to be SVP_E_UNSUPPORTED; they are now
    accepted and match as their own group (the plain-load kernel)."""
    with svp.Context(dry_run=True) as c:
        sg = c.register_kernel("sgemm")
        shapes = [(64, 64, 64, 0), (64, 130, 64, 0), (64, 64, 30, 0), (64, 64, 64, 4), (33, 17, 5, 0)]
        for vp, (M, N, K, off) in enumerate(shapes):
            base = FAKE + vp * 2**34
            c.submit(vp, sg, svp.args_sgemm(M, N, K), [(base + off, 4 * M * K, svp.DIR_IN, 0),
                                                       (base + 2**30, 4 * K * N, svp.DIR_IN, 0),
                                                       (base + 2**31, 4 * M * N, svp.DIR_OUT, 0)])
        c.flush()
        ops = [op for op in c.plan() if op["kind"] == svp.OP_KERNEL]
        assert sorted(sorted(op["vps"]) for op in ops) == [[0], [1, 2, 3, 4]]


def test_zero_sized_jobs_are_legal():
    with svp.Context(dry_run=True) as c:
        va = c.register_kernel("vecadd")
        c.submit(0, va, svp.args_vecadd(0), [(0, 0, 1, 0), (0, 0, 1, 0), (0, 0, 2, 0)])
        c.flush()
        assert c.flush_stats()["jobs"] == 1


def test_batch_is_all_or_nothing():
    with svp.Context(dry_run=True) as c:
        va = c.register_kernel("vecadd")
        good = (0, va, svp.args_vecadd(10), _vecadd_bufs(10))
        bad = (1, va, svp.args_vecadd(10), _vecadd_bufs(10)[:2])
        with pytest.raises(svp.SvpError):
            c.submit_batch([good, bad])
        c.flush()
        assert c.flush_stats()["jobs"] == 0
        ids = c.submit_batch([good, (1, va, svp.args_vecadd(10), _vecadd_bufs(10))])
        assert ids[1] == ids[0] + 1


def test_thread_safe_concurrent_submit():
    from concurrent.futures import ThreadPoolExecutor
    with svp.Context(dry_run=True) as c:
        va = c.register_kernel("vecadd")

        def worker(vp):
            for _ in range(50):
                c.submit(vp, va, svp.args_vecadd(100), _vecadd_bufs(100))

        with ThreadPoolExecutor(8) as ex:
            list(ex.map(worker, range(16)))
        c.flush()
        st = c.flush_stats()
        assert st["jobs"] == 800 and st["levels"] == 50
        assert st["launches"] == 50  # one coalesced launch per level


def test_lpt_partition_pure():
    out = svp.lpt_partition([1, 1, 1, 1], [5.0, 5.0, 5.0, 5.0], 2)
    assert out == [0, 1, 0, 1]
    with pytest.raises(svp.SvpError):
        svp.lpt_partition([1], [1.0], 0)


_STRUCTS = ("svp_config", "svp_buf", "svp_job_desc", "svp_ipc_buf", "svp_vp_profile", "svp_kernel_stats",
            "svp_flush_stats", "svp_plan_op", "svp_device_stats")


def test_ctypes_layouts_match_the_header(tmp_path):
    """The binding's ctypes mirrors have the C compiler's size and field offsets (a field
    added to the header but not to svp.py -- or vice versa -- fails here)."""
    import ctypes
    import shutil
    import subprocess
    if not shutil.which("gcc"):
        pytest.skip("gcc not available")
    lines = ["#include <stdio.h>", "#include <stddef.h>", '#include "svp.h"', "int main(void) {"]
    for name in _STRUCTS:
        py = getattr(svp, name)
        lines.append(f'printf("{name} %zu\\n", sizeof({name}));')
        for f, _ in py._fields_:
            lines.append(f'printf("{name}.{f} %zu\\n", offsetof({name}, {f}));')
    lines.append("return 0; }")
    src = tmp_path / "layout.c"
    src.write_text("\n".join(lines))
    exe = tmp_path / "layout"
    subprocess.run(["gcc", "-std=c11", "-I", os.path.join(ROOT, "include"), str(src), "-o", str(exe)], check=True)
    got = dict(l.split() for l in subprocess.run([str(exe)], check=True, capture_output=True, text=True).stdout.splitlines())
    for name in _STRUCTS:
        py = getattr(svp, name)
        assert int(got[name]) == ctypes.sizeof(py), name
        for f, _ in py._fields_:
            assert int(got[f"{name}.{f}"]) == getattr(py, f).offset, f"{name}.{f}"


def test_ew_mix_id_is_stats_only():
    with svp.Context(dry_run=True) as c:
        assert c.kernel_stats(svp.KERNEL_EW_MIX)["launches"] == 0
        with pytest.raises(svp.SvpError) as e:
            c.submit(0, svp.KERNEL_EW_MIX, svp.args_vecadd(4), _vecadd_bufs(4))
        assert e.value.status == svp.SVP_E_NOKERNEL


def test_table_mode_values():
    with svp.Context(dry_run=True, table_mode=svp.TABLE_PARAM):
        pass
    with pytest.raises(svp.SvpError) as e:
        svp.Context(dry_run=True, table_mode=2)
    assert e.value.status == svp.SVP_E_INVAL


def test_use_after_finalize_and_null_context():
    """after svp_finalize the binding holds no handle, and every entry point
    answers a null context with SVP_E_INVAL (no crash, no CUDA call)."""
    c = svp.Context(dry_run=True)
    k = c.register_kernel("vecadd")
    c.close()
    c.close()  # idempotent
    for call in (lambda: c.flush(), lambda: c.profile(-1), lambda: c.flush_stats(), lambda: c.reset_profile(),
                 lambda: c.submit(0, k, svp.args_vecadd(0), [(0, 0, 1, 0)] * 2 + [(0, 0, 2, 0)]),
                 lambda: c.register_kernel("saxpy"), lambda: c.vp_device(0)):
        with pytest.raises(svp.SvpError) as e:
            call()
        assert e.value.status == svp.SVP_E_INVAL
    L = svp.load()
    assert L.svp_flush(None) == svp.SVP_E_INVAL
    assert L.svp_finalize(None) in (svp.SVP_OK, svp.SVP_E_INVAL)


def test_host_alloc_rejects_dry_run_and_bad_args():
    """svp_host_alloc needs CUDA (page-locking); a dry-run context answers UNSUPPORTED, and
    argument errors / unknown pointers answer INVAL without touching the allocator."""
    with svp.Context(dry_run=True) as c:
        with pytest.raises(svp.SvpError) as e:
            c.host_alloc(0, 4096)
        assert e.value.status == svp.SVP_E_UNSUPPORTED
        with pytest.raises(svp.SvpError) as e:
            c.host_alloc(0, 0)
        assert e.value.status == svp.SVP_E_INVAL
        with pytest.raises(svp.SvpError) as e:
            c.host_alloc(5, 4096)
        assert e.value.status == svp.SVP_E_INVAL
        with pytest.raises(svp.SvpError) as e:
            c.host_free(0x1000)
        assert e.value.status == svp.SVP_E_INVAL


def test_flush_async_tickets_dry_run():
    """svp_flush_async / svp_flush_wait bookkeeping without a GPU: tickets count flushes,
    a dry-run flush completes at once, svp_wait sees its jobs done, unknown tickets are
    rejected."""
    with svp.Context(dry_run=True) as c:
        k = c.register_kernel("vecadd")
        buf = [(0x10000, 4096, svp.DIR_IN, svp.MEM_DEVICE), (0x20000, 4096, svp.DIR_IN, svp.MEM_DEVICE),
               (0x30000, 4096, svp.DIR_OUT, svp.MEM_DEVICE)]
        tickets = []
        for r in range(3):
            ids = c.submit_batch([(0, k, svp.args_vecadd(1024), buf)])
            tickets.append(c.flush_async())
            c.wait(ids[0])
        assert tickets == [tickets[0], tickets[0] + 1, tickets[0] + 2]
        c.flush_wait(tickets[-1])
        c.flush()  # a synchronous flush takes the next ticket
        with pytest.raises(svp.SvpError) as e:
            c.flush_wait(tickets[-1] + 10)
        assert e.value.status == svp.SVP_E_INVAL
