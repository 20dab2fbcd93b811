"""Timing models and brute-force schedules (TEST INFRASTRUCTURE ONLY; see oracle/__init__.py).

Everything here is the plain statement of a formula the paper prints or of the
textbook definition our DESIGN.md reading of the paper adopts:

* Eq 7 (§5 "Kernel Interleaving"):  T_total = 2 Tm + N max(Tm, Tk)
* Eq 8:                            Speedup = 3N / (2 + N)
* Eq 9 (garbled ``d...e`` read as a ceiling):
                                                         T = To + Te * ceil(xi / lambda)
* The Copy/Compute engine model of Fig 3: a job is
  H2D copy -> kernel -> D2H copy, each engine serves one op at a time, in the order
  given -- i.e. a 3-machine permutation flow shop.  ``flowshop_makespan`` is its
  textbook recurrence; ``best_makespan`` is brute force over all orders.
* The Re-scheduler's order (the paper cites "a non-preemptive, optimal scheduler
  augmented for job dependencies [14]" without giving it):
  DESIGN.md reading R4 = Johnson's rule on (Tin + Tk, Tk + Tout).  ``johnson_order``
  is Johnson's 1954 rule written out.
* The Job Dispatcher's VP->GPU placement (reading R1/§8(e)): LPT (longest
  processing time first, least-loaded GPU) and the brute-force optimal partition.

Profiler attribution inside one coalesced launch (a VP's share of one kernel's
device time) has no reference value anywhere: **parity unpinned**; only the
conservation law (shares sum to the measured time) is checked.
"""
from __future__ import annotations

import itertools
import math
from typing import List, Sequence, Tuple


def eq7_total(N: int, Tm: float, Tk: float) -> float:
    """Makespan of N interleaved H2D->kernel->D2H programs, Eq 7."""
    return 2.0 * Tm + N * max(Tm, Tk)


def eq8_speedup(N: int) -> float:
    """Interleaving speedup for Tk = Tm, Eq 8."""
    return 3.0 * N / (2.0 + N)


def eq9_time(To: float, Te: float, xi: float, lam: float) -> float:
    """Kernel time from the aligned processing unit lambda, Eq 9."""
    return To + Te * math.ceil(xi / lam)


def serial_time(jobs: Sequence[Tuple[float, float, float]]) -> float:
    """No interleaving: every op waits for the previous one ("3N")."""
    return float(sum(a + b + c for a, b, c in jobs))


def flowshop_makespan(jobs: Sequence[Sequence[float]], order: Sequence[int] | None = None) -> float:
    """Permutation flow shop: C[j][m] = max(C[j-1][m], C[j][m-1]) + p[j][m]."""
    order = list(range(len(jobs))) if order is None else list(order)
    if not order:
        return 0.0
    nm = len(jobs[0])
    done = [0.0] * nm
    for j in order:
        prev = 0.0
        for m in range(nm):
            start = max(done[m], prev)
            done[m] = start + jobs[j][m]
            prev = done[m]
    return done[-1]


def best_makespan(jobs: Sequence[Sequence[float]]) -> float:
    """Brute force over all permutations (tiny N only)."""
    return min(flowshop_makespan(jobs, p) for p in itertools.permutations(range(len(jobs))))


def johnson_order(jobs: Sequence[Sequence[float]]) -> List[int]:
    """Johnson's rule.  For 2 stages (a, b): jobs with a < b first in ascending a, then
    the rest in descending b.  For 3 stages (a, b, c) use the surrogate
    (a + b, b + c) (reading R4).  Ties keep the lower index first."""
    if len(jobs) and len(jobs[0]) == 3:
        pairs = [(a + b, b + c) for a, b, c in jobs]
    else:
        pairs = [(a, b) for a, b in jobs]
    first = sorted([i for i, (a, b) in enumerate(pairs) if a < b], key=lambda i: (pairs[i][0], i))
    last = sorted([i for i, (a, b) in enumerate(pairs) if a >= b], key=lambda i: (-pairs[i][1], i))
    return first + last


def lpt_partition(costs: Sequence[float], G: int) -> List[int]:
    """LPT: largest cost first (ties: lower index), each to the least-loaded GPU
    (ties: lower GPU id).  Returns the GPU of every item."""
    load = [0.0] * G
    out = [0] * len(costs)
    for i in sorted(range(len(costs)), key=lambda i: (-costs[i], i)):
        g = min(range(G), key=lambda g: (load[g], g))
        out[i] = g
        load[g] += costs[i]
    return out


def partition_makespan(costs: Sequence[float], assign: Sequence[int], G: int) -> float:
    load = [0.0] * G
    for c, g in zip(costs, assign):
        load[g] += c
    return max(load) if load else 0.0


def best_partition_makespan(costs: Sequence[float], G: int) -> float:
    """Brute-force optimal makespan over all G^n assignments (tiny n only)."""
    best = math.inf
    for assign in itertools.product(range(G), repeat=len(costs)):
        best = min(best, partition_makespan(costs, assign, G))
    return best


def graham_bound(G: int) -> float:
    """LPT <= (4/3 - 1/(3G)) OPT (Graham 1969)."""
    return 4.0 / 3.0 - 1.0 / (3.0 * G)
