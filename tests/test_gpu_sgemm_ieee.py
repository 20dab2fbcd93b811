"""IEEE edge values through every fp32 "sgemm" implementation (DESIGN.md
R20): +-Inf, NaN (incl. a payload only in the low 13 bits and the all-ones pattern), values
at FLT_MAX and at the TF32 rounding boundary, subnormal operands (alone, and times large
operands so the products are normal), against the oracle (fp64 IEEE accumulation, one
rounding), with alpha / beta, in one coalesced launch of two VPs.  NaN / +-Inf positions
must match exactly; finite outputs meet the stated bound (ieee_cases.STATED)."""
import numpy as np
import pytest

import oracle
import workloads as W
from gpu_common import run_svp
from ieee_cases import STATED, compare, edge_inputs, passed
from paper_conf_dac_jungc15_b200 import svp

pytestmark = pytest.mark.gpu

IMPLS = {"ffma": svp.SGEMM_FFMA, "3xtf32": svp.SGEMM_3XTF32, "tf32bf16": svp.SGEMM_TF32BF16}


@pytest.mark.parametrize("impl", list(IMPLS))
@pytest.mark.parametrize("beta", [0.0, 0.5])
@pytest.mark.parametrize("shape", [(256, 256, 64), (1024, 1024, 256), (200, 136, 72)])
def test_ieee_edge_values(impl, beta, shape):
    M, N, K = shape
    alpha = -1.5 if beta else 1.0
    specs = [W.JobSpec(v, "sgemm", M=M, N=N, K=K, alpha=alpha, beta=beta) for v in range(2)]
    inputs = [edge_inputs(M, N, K, seed=21 + v, beta=beta) for v in range(2)]
    outs, _, _ = run_svp(specs, inputs, "device", sgemm_impl=IMPLS[impl])
    for s, inp, got in zip(specs, inputs, outs):
        O = oracle.sgemm(inp["A"], inp["B"], inp.get("C"), s.alpha, s.beta)
        r = compare(got["C"], O, inp["A"], inp["B"], s.alpha, s.beta, inp.get("C"), **STATED[impl])
        assert passed(r), (impl, s.vp, r)
        # the exact probes: a subnormal operand times 2^120 is not flushed, Inf*Inf = Inf
        assert got["C"][12, 12] == O[12, 12], (impl, got["C"][12, 12], O[12, 12])
        assert np.isinf(O[5, 6]) and got["C"][5, 6] == O[5, 6]
