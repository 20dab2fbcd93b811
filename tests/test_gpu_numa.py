"""NUMA placement of host-resident VP buffers and per-GPU worker threads (ABI 6:
svp_host_alloc / svp_host_free, svp_device_stats.numa_node / worker_cpu_pinned).

The expected node and CPUs come from the kernel, not from libsvp: sysfs of the GPU's PCI
function (as torch reports its bus id) and /proc/self/numa_maps for where the pages'
policy points."""
import os

import pytest
import torch

import workloads as W
from gpu_common import check_job, inputs_for
from paper_conf_dac_jungc15_b200 import svp
from paper_conf_dac_jungc15_b200.vpset import VPSet

pytestmark = pytest.mark.gpu


def _pci_dir(ordinal):
    p = torch.cuda.get_device_properties(ordinal)
    dom, bus, dev = (getattr(p, k, None) for k in ("pci_domain_id", "pci_bus_id", "pci_device_id"))
    if bus is None:
        return None
    return "/sys/bus/pci/devices/%04x:%02x:%02x.0" % (dom or 0, bus, dev or 0)


def _sysfs_node(ordinal):
    d = _pci_dir(ordinal)
    try:
        with open(os.path.join(d, "numa_node")) as f:
            return int(f.read().strip())
    except (TypeError, OSError, ValueError):
        return -1


def _sysfs_cpus(ordinal):
    d = _pci_dir(ordinal)
    try:
        with open(os.path.join(d, "local_cpulist")) as f:
            txt = f.read().strip()
    except (TypeError, OSError):
        return set()
    cpus = set()
    for part in filter(None, txt.split(",")):
        a, _, b = part.partition("-")
        cpus.update(range(int(a), int(b or a) + 1))
    return cpus


def _policy_of(addr):
    with open("/proc/self/numa_maps") as f:
        for line in f:
            if int(line.split()[0], 16) == addr:
                return line.split()[1]
    return None


def test_host_alloc_places_pages_on_the_gpus_node():
    want = _sysfs_node(0)
    with svp.Context(num_gpus=1) as ctx:
        addr, node = ctx.host_alloc(0, (8 << 20) + 123)
        assert addr % 4096 == 0
        assert node == want or (node == -1 and want < 0), (node, want)
        assert ctx.device_stats(0)["numa_node"] == want
        if node >= 0:
            assert _policy_of(addr) == f"prefer:{node}"
        # page-locked: a DMA copy both ways through it (torch over the same bytes)
        import ctypes
        host = torch.frombuffer((ctypes.c_uint8 * (8 << 20)).from_address(addr), dtype=torch.uint8)
        src = torch.arange(8 << 20, dtype=torch.int64, device="cuda").to(torch.uint8)
        host.copy_(src, non_blocking=True)
        torch.cuda.synchronize()
        assert torch.equal(host.cuda(), src)
        ctx.host_free(addr)
        with pytest.raises(svp.SvpError) as e:
            ctx.host_free(addr)
        assert e.value.status == svp.SVP_E_INVAL
        ctx.host_alloc(0, 4096)  # left for svp_finalize to release


def test_host_numa_vpset_parity():
    """Host-resident VPs on svp_host_alloc blocks: submit accepts them as HOST_PINNED and every
    VP's output matches the oracle; a released block is not accepted from the range cache."""
    specs = W.mixed_small(nvps=24, max_n=70000)
    inputs = inputs_for(specs)
    with svp.Context(num_gpus=1, profile_level=1) as ctx:
        vs = VPSet(ctx, specs, inputs, "host", host_numa=True)
        assert len(vs.host_blocks) == sum(len(r) for r in vs.raw)
        vs.submit()
        ctx.flush()
        for i, (s, inp) in enumerate(zip(specs, inputs)):
            check_job(s, inp, vs.output(i))
        assert vs.guards_intact()
        jobs = [j for j, s in zip(vs.job_list(), specs) if s.n > 0]  # (empty jobs touch nothing)
        vs.release_host()
        with pytest.raises(svp.SvpError) as e:
            ctx.submit_batch(jobs[:1])
        assert e.value.status == svp.SVP_E_INVAL


@pytest.mark.parametrize("affinity", ["1", "0"])
def test_worker_threads_pinned_near_their_gpu(small_specs, affinity, monkeypatch):
    """GPU index 1's worker thread runs on GPU 1's local CPUs (two logical GPUs on ordinal 0
    here); SVP_NUMA_AFFINITY=0 leaves it unpinned.  GPU 0 is the flushing thread's."""
    monkeypatch.setenv("SVP_NUMA_AFFINITY", affinity)
    local = _sysfs_cpus(0) & os.sched_getaffinity(0)
    specs, inputs = small_specs
    with svp.Context(num_gpus=2, device_ids=[0, 0], profile_level=1) as ctx:
        ds = [ctx.device_stats(g) for g in range(2)]
        assert ds[0]["worker_cpu_pinned"] == 0
        assert ds[1]["worker_cpu_pinned"] == (1 if (affinity == "1" and local) else 0), (ds, local)
        assert ds[0]["numa_node"] == ds[1]["numa_node"] == _sysfs_node(0)
        vs = VPSet(ctx, specs, inputs, "host", device_ordinals=[0, 0], host_numa=True)
        vs.submit()
        ctx.flush()
        for i, (s, inp) in enumerate(zip(specs, inputs)):
            check_job(s, inp, vs.output(i))
        assert {op["device"] for op in ctx.plan()} == {0, 1}


@pytest.fixture(scope="module")
def small_specs():
    specs = W.mixed_small(nvps=16, max_n=40000)
    return specs, inputs_for(specs)
