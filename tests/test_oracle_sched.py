"""Pins for oracle.sched: the paper's timing models and the brute-force schedules."""
import itertools
import math

import numpy as np
import pytest

from oracle import sched


def test_eq8_values_from_paper(golden):
    for row in golden("paper_models.txt"):
        if row[0] == "eq8":
            N, s = int(row[1]), float(row[2])
            assert sched.eq8_speedup(N) == pytest.approx(s, rel=1e-15)
    # "about 3x for large N"
    assert 2.99 < sched.eq8_speedup(10_000) < 3.0


def test_eq8_is_eq7_ratio_when_tk_equals_tm():
    # Eq 8 follows from Eq 7 with Tk = Tm = T and a serial time of 3NT
    for N in (1, 2, 5, 32):
        T = 1.7
        assert sched.serial_time([(T, T, T)] * N) / sched.eq7_total(N, T, T) == pytest.approx(sched.eq8_speedup(N))


@pytest.mark.parametrize("N", [1, 2, 3, 8, 17])
def test_eq7_vs_three_engine_pipeline(N):
    """Eq 7 is exact for the 3-engine pipeline when Tk >= Tm and over-predicts by
    (Tm - Tk) otherwise (SURVEY §8c.3 "Interleave timing")."""
    Tm = 13.44  # Fig 9(a) memcpy time, ms
    for Tk in np.linspace(0.0, 60.0, 31):
        sim = sched.flowshop_makespan([(Tm, Tk, Tm)] * N)
        eq7 = sched.eq7_total(N, Tm, Tk)
        if Tk >= Tm:
            assert sim == pytest.approx(eq7)
        else:
            assert eq7 - sim == pytest.approx(Tm - Tk)


def test_fig9a_speedup_peaks_at_tk_equals_tm():
    Tm = 13.44
    ks = np.linspace(0.5, 100, 400)
    sp = [sched.serial_time([(Tm, k, Tm)] * 2) / sched.eq7_total(2, Tm, k) for k in ks]
    assert abs(ks[int(np.argmax(sp))] - Tm) < 0.5


def test_eq9_staircase_grid9_equals_grid16(golden):
    row = [r for r in golden("paper_models.txt") if r[0] == "eq9"][0]
    kv = dict(x.split("=") for x in row[1:])
    thr, lam = int(kv["threads"]), int(kv["lambda_blocks"]) * int(kv["threads"])
    t9 = sched.eq9_time(1.0, 2.0, int(kv["grid_a"]) * thr, lam)
    t16 = sched.eq9_time(1.0, 2.0, int(kv["grid_b"]) * thr, lam)
    t17 = sched.eq9_time(1.0, 2.0, 17 * thr, lam)
    assert t9 == t16 < t17


def test_flowshop_recurrence_by_hand():
    jobs = [(3, 2, 1), (1, 4, 2)]
    # order 0,1: M1 0-3, 3-4; M2 3-5, 5-9; M3 5-6, 9-11
    assert sched.flowshop_makespan(jobs, [0, 1]) == 11
    # order 1,0: M1 0-1, 1-4; M2 1-5, 5-7; M3 5-7, 7-8
    assert sched.flowshop_makespan(jobs, [1, 0]) == 8
    assert sched.best_makespan(jobs) == 8


@pytest.mark.parametrize("seed", range(40))
def test_johnson_two_machine_is_optimal(seed):
    g = np.random.default_rng(seed)
    n = int(g.integers(1, 8))
    jobs = [tuple(map(float, g.integers(1, 20, 2))) for _ in range(n)]
    o = sched.johnson_order(jobs)
    assert sorted(o) == list(range(n))
    assert sched.flowshop_makespan(jobs, o) == pytest.approx(sched.best_makespan(jobs))


@pytest.mark.parametrize("seed", range(40))
def test_johnson_three_machine_dominated_is_optimal(seed):
    """Johnson's 3-machine condition: min(a) >= max(b) (copy-bound jobs)."""
    g = np.random.default_rng(100 + seed)
    n = int(g.integers(1, 7))
    jobs = [(float(g.integers(10, 30)), float(g.integers(0, 10)), float(g.integers(10, 30))) for _ in range(n)]
    o = sched.johnson_order(jobs)
    assert sched.flowshop_makespan(jobs, o) == pytest.approx(sched.best_makespan(jobs))


@pytest.mark.parametrize("G", [2, 3, 4])
def test_lpt_within_graham_bound(G):
    g = np.random.default_rng(G)
    for _ in range(25):
        costs = list(map(float, g.integers(1, 50, int(g.integers(1, 9)))))
        a = sched.lpt_partition(costs, G)
        assert all(0 <= x < G for x in a)
        got = sched.partition_makespan(costs, a, G)
        opt = sched.best_partition_makespan(costs, G)
        assert opt <= got <= sched.graham_bound(G) * opt + 1e-9


def test_lpt_tie_breaks():
    assert sched.lpt_partition([5, 5, 5, 5], 2) == [0, 1, 0, 1]
    assert sched.lpt_partition([1, 9, 3], 2) == [1, 0, 1]
