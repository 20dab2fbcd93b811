"""N>1 path on CPU: world_size-2 gloo processes, each a 'rank' of the Job Dispatcher.

Every rank computes the same kernel-stratified LPT partition (svp_lpt_partition, no
data exchange), keeps its VPs, and plans them in a dry-run context; the ranks then
all_gather_object their VP sets and plan summaries to check the partition is exact
(disjoint, covering), balanced per kernel class, and that no rank's plan touches
another rank's VP.  This is bench.py's --gpus N code path (bench.my_specs)."""
import os
import socket

import pytest
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


FAKE = 0x7F0000000000


def _worker(rank, ws, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank), WORLD_SIZE=str(ws))
    dist.init_process_group("gloo", rank=rank, world_size=ws)
    try:
        import bench
        import workloads as W
        from paper_conf_dac_jungc15_b200 import svp
        from paper_conf_dac_jungc15_b200.vpset import BUFS, job_args, buffer_elems
        specs = W.config_specs(5)
        mine = bench.my_specs(specs, rank, ws)
        ctx = svp.Context(dry_run=True)
        jobs = []
        for s in mine:
            kid = ctx.kernel(s.kernel)
            bl = []
            for b, (name, dt, d) in enumerate(BUFS[s.kernel]):
                es = 1 if dt == "u8" else 4
                nb = buffer_elems(s, name) * es
                bl.append((FAKE + s.vp * (1 << 36) + b * (1 << 33), nb, d, 0))
            jobs.append((s.vp, kid, job_args(s), bl))
        ctx.submit_batch(jobs)
        ctx.flush()
        plan_vps = sorted(v for op in ctx.plan() for v in op["vps"])
        st = ctx.flush_stats()
        ctx.close()
        out = [None] * ws
        dist.all_gather_object(out, {"vps": sorted(s.vp for s in mine), "plan_vps": plan_vps,
                                     "groups": st["groups"], "kinds": sorted(s.kernel for s in mine)})
        if rank == 0:
            q.put(out)
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("ws", [2])
def test_two_rank_dispatch_partition(ws):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, ws, port, q)) for r in range(ws)]
    for p in procs:
        p.start()
    res = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    allv = [v for r in res for v in r["vps"]]
    assert sorted(allv) == list(range(256)) and len(set(allv)) == 256   # disjoint + covering
    for r in res:
        assert r["plan_vps"] == r["vps"]                                 # a rank plans only its VPs
        assert r["groups"] == 5                                          # every rank keeps every class
    for k in ("vecadd", "saxpy", "hist256", "blackscholes", "sgemm"):
        counts = [r["kinds"].count(k) for r in res]
        assert max(counts) - min(counts) <= 1
