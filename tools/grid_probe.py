"""Resident CTAs per SM of the memory-bound launches vs time and power (energy-bound GPU:
fewer resident warps may move the same bytes for less power).  argv: subset label;
SVP_EW_PER_SM / SVP_BS_PER_SM set by the caller.  Prints one JSON line per subset."""
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))
import workloads as W  # noqa: E402
from overlap_probe import run  # noqa: E402

torch.cuda.set_device(0)
specs = W.config_specs(5)
inputs = W.make_inputs_many(specs)
subsets = {"vecadd": ["vecadd"], "blackscholes": ["blackscholes"], "membound": list(W.MEMBOUND),
           "all": list(W.KERNELS)}
for name in sys.argv[1].split(","):
    idx = [i for i, s in enumerate(specs) if s.kernel in subsets[name]]
    r = run(name, [specs[i] for i in idx], [inputs[i] for i in idx], long_s=1.5)
    print("RESULT", json.dumps({"subset": name, "ew_per_sm": os.environ.get("SVP_EW_PER_SM", "max"),
                                "bs_per_sm": os.environ.get("SVP_BS_PER_SM", "max"), **r}), flush=True)
