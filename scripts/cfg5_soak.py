"""Full-size cfg5 soak: the bench's launch configuration (plus the hetero / graph / table
options) flushed for several steps, every memory-bound VP checked against the oracle after
every step (SAXPY chained on its previous output), every SGEMM VP on 8 sampled elements.
argv: steps, then option sets as hetero:graph:table[:interleave] (e.g. 0:0:1 1:1:1 0:1:0:0;
interleave 0 = one stream, where Black-Scholes / mixed launches take the dynamic tile
order).  GPU tool."""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
sys.path.insert(0, "tests")
import oracle  # noqa: E402
import workloads as W  # noqa: E402
from gpu_common import check_job  # noqa: E402
from paper_conf_dac_jungc15_b200 import svp  # noqa: E402
from paper_conf_dac_jungc15_b200.vpset import VPSet  # noqa: E402

steps = int(sys.argv[1])
combos = [tuple(int(x) for x in (c + ":1").split(":")[:4]) for c in sys.argv[2:]] or [(0, 0, 1, 1)]
specs = W.config_specs(5)
inputs = W.make_inputs_many(specs)
mb = [i for i, s in enumerate(specs) if s.kernel != "sgemm"]
g = np.random.default_rng(11)
stream = torch.cuda.current_stream()
for hetero, graph, table, inter in combos:
    ctx = svp.Context(num_gpus=1, device_ids=[0], profile_level=1, external_streams=[stream.cuda_stream],
                      hetero=bool(hetero), graph=bool(graph), table_mode=table, interleave=bool(inter))
    vs = VPSet(ctx, specs, inputs, "device", device_ordinals=[0])
    jobs = svp.JobBatch(vs.job_list())
    prev = [dict(inp) for inp in inputs]
    bad = 0
    for step in range(steps):
        ctx.submit_batch(jobs)
        ctx.flush()
        torch.cuda.synchronize()
        want = oracle.run_jobs([specs[i] for i in mb], [prev[i] for i in mb])
        for i, w in zip(mb, want):
            got = vs.output(i)
            try:
                check_job(specs[i], prev[i], got, w)
            except AssertionError as e:
                bad += 1
                print(f"combo {hetero}:{graph}:{table} step {step} vp {specs[i].vp} {specs[i].kernel}: {e}", flush=True)
            if specs[i].kernel == "saxpy":
                prev[i] = dict(prev[i], y=got["y"].copy())
        for i, s in enumerate(specs):
            if s.kernel == "sgemm":
                smp = [(int(g.integers(0, s.M)), int(g.integers(0, s.N))) for _ in range(8)]
                try:
                    check_job(s, inputs[i], vs.output(i), sample=smp)
                except AssertionError as e:
                    bad += 1
                    print(f"combo {hetero}:{graph}:{table} step {step} vp {s.vp} sgemm: {e}", flush=True)
    st = ctx.flush_stats()
    print(f"combo hetero={hetero} graph={graph} table={table} interleave={inter}: {bad} bad over {steps} steps; "
          f"graph_replays {st['graph_replays']} guards {vs.guards_intact()}", flush=True)
    ctx.close()
    del vs
    torch.cuda.empty_cache()
