"""bench.py host logic on CPU (no GPU): the L2 rotation, the GPU plan for --gpus N (one
process driving N GPUs, or one rank per GPU), and the Job Dispatcher's split of BASELINE
cfg5's 256 VPs over 2 GPUs in a dry-run context (the placement bench.py then drives)."""
import importlib.util
import os
import types

import pytest

import workloads as W
from paper_conf_dac_jungc15_b200 import svp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _bench():
    spec = importlib.util.spec_from_file_location("bench_mod", os.path.join(ROOT, "bench.py"))
    m = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(m)
    return m


def test_buffer_sets_cover_four_times_l2():
    b = _bench()
    for cfg, want in ((1, 21), (2, 11), (3, 1), (4, 1), (5, 1)):
        specs = W.config_specs(cfg)
        n = b.n_buffer_sets(specs)
        assert n == want, (cfg, n)
        ws = sum(s.input_bytes() + s.output_bytes() for s in specs)
        assert n * ws >= 4 * b.L2_BYTES or n == 1 and ws >= 4 * b.L2_BYTES


def test_gpu_plan_single_process_and_ranks(monkeypatch):
    b = _bench()
    import torch
    monkeypatch.setattr(torch.cuda, "device_count", lambda: 8)
    args = types.SimpleNamespace(gpus=4)
    monkeypatch.delenv("SVP_BENCH_DEVICES", raising=False)
    assert b.gpu_plan(args, 1, 0) == ([0, 1, 2, 3], "single")
    assert b.gpu_plan(args, 4, 2) == ([2], "process")
    with pytest.raises(SystemExit):
        b.gpu_plan(args, 2, 0)  # WORLD_SIZE must equal --gpus
    monkeypatch.setenv("SVP_BENCH_DEVICES", "0,0,0,0")
    assert b.gpu_plan(args, 1, 0) == ([0, 0, 0, 0], "single")
    monkeypatch.setattr(torch.cuda, "device_count", lambda: 1)
    monkeypatch.delenv("SVP_BENCH_DEVICES")
    with pytest.raises(SystemExit):
        b.gpu_plan(args, 1, 0)  # 4 GPUs asked, 1 present, no logical mapping: refuse


@pytest.mark.parametrize("G", [2, 4, 8])
def test_cfg5_dispatcher_split(G):
    """bench.py --gpus G (strong scaling): the 256 cfg5 VPs are placed by the library's
    kernel-stratified LPT (VPSet's costs), every GPU gets a share of every kernel class and
    the VP counts differ by at most one per class."""
    specs = W.config_specs(5)
    with svp.Context(dry_run=True, num_gpus=G) as c:
        kids = {k: c.kernel(k) for k in W.KERNELS}
        costs = [float(s.algorithmic_bytes()) / 6550.0 + float(s.flops()) / 4.0e5 for s in specs]
        dev = c.assign_vps([s.vp for s in specs], [kids[s.kernel] for s in specs], costs)
        ds = [c.device_stats(g) for g in range(G)]
    assert sum(d["vps"] for d in ds) == 256
    for k in W.KERNELS:
        per = [sum(1 for s, d in zip(specs, dev) if s.kernel == k and d == g) for g in range(G)]
        assert min(per) >= 1, (k, per)  # every GPU coalesces a share of every class
        cl = [sum(c for s, c, d in zip(specs, costs, dev) if s.kernel == k and d == g) for g in range(G)]
        items = [c for s, c in zip(specs, costs) if s.kernel == k]
        assert max(cl) <= sum(items) / G + max(items) + 1e-6, (k, cl)  # list-scheduling bound
    if G == 2:
        assert abs(ds[0]["vps"] - ds[1]["vps"]) <= 4, [d["vps"] for d in ds]
    loads = [d["est_load_ns"] for d in ds]
    assert max(loads) / (sum(loads) / G) < 1.15
