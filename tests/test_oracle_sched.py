"""Pins for oracle.sched (Fig. 10, Eq. 4-18), none of which re-derives the oracle from itself:
- a hand-worked run of Fig. 10 on the paper's own test system (tests/golden/fig10_paper_system.txt);
- the D/D/1 queue recursion (Lindley) for a single partition with no deadline pressure;
- the closed-form step-5 choice when every partition meets the deadline;
- step 6 (earliest response) when no partition can meet it;
- Eq. 4's range split and Eq. 7/10/14 values printed in the paper."""
import math
import os

import numpy as np
import pytest

from oracle import sched

HERE = os.path.dirname(os.path.abspath(__file__))

# the paper's performance functions
EQ10 = (512.0, 6e-5, 0.984, 0.0, 4e-5, 1.0, 0.0146)
EQ14 = {1: (math.inf, 0.003, 1.0, 0.0258, 0, 1, 0), 2: (math.inf, 0.0015, 1.0, 0.013, 0, 1, 0),
        4: (math.inf, 0.0008, 1.0, 0.0065, 0, 1, 0)}
EQ15 = (math.inf, 0.00021, 1.0, 0.0020, 0, 1, 0)


def paper_partitions():
    return ([(sched.CUBE, False, EQ10)] +
            [(sched.TABLE, True, EQ14[k]) for k in (1, 1, 2, 2, 4, 4)])


def load_golden():
    events = []
    for line in open(os.path.join(HERE, "golden", "fig10_paper_system.txt")):
        line = line.strip()
        if not line or line.startswith("#"):
            continue
        if line.startswith("C"):
            _, p, est, real = line.split()
            events.append(("C", int(p), float(est), float(real)))
        else:
            lhs, rhs = line.split("|")
            _, t, mb, cf, tt = lhs.split()
            p, tr, r = rhs.split()
            events.append(("Q", float(t), float(mb), float(cf), float(tt), int(p), int(tr), float(r)))
    return events


def test_fig10_hand_worked_paper_system():
    s = sched.Fig10(paper_partitions(), 0.020)
    n = 0
    for ev in load_golden():
        if ev[0] == "C":
            s.complete(ev[1], ev[2], ev[3])
            continue
        _, t, mb, cf, tt, p, tr, r = ev
        got = s.submit(t, mb, cf, tt)
        assert got[0] == p and got[1] == tr, (n, got, ev)
        assert abs(got[2] - r) < 5e-7, (n, got, ev)
        assert got[3] == pytest.approx(t + 0.020)
        n += 1
    assert n == 13


def test_paper_printed_functions():
    # Eq. 10 range A and B, Eq. 14/15 at C/C_TOT = 1
    assert sched.perf(EQ10, 100.0) == pytest.approx(6e-5 * 100 ** 0.984)
    assert sched.perf(EQ10, 1024.0) == pytest.approx(4e-5 * 1024 + 0.0146)
    assert sched.perf(EQ10, 512.0) == pytest.approx(4e-5 * 512 + 0.0146)  # R25: 512 MB is range B
    assert sched.perf(EQ14[4], 1.0) == pytest.approx(0.0073)
    assert sched.perf(EQ15, 0.5) == pytest.approx(0.002105)
    # a 14-SM GPU is faster than any single partition of it (Eq. 15 vs Eq. 14)
    for x in (0.1, 0.5, 1.0):
        assert sched.perf(EQ15, x) < min(sched.perf(EQ14[k], x) for k in (1, 2, 4))
    # Eq. 17-18: 13.8 ns per dictionary entry, summed over the text conditions
    assert sched.trans_upper_bound([52, 100, 128, 1826]) == pytest.approx(2106 * 13.8e-9)


def test_single_partition_is_a_fifo_queue():
    """One TABLE partition and no deadline pressure: T_R follows the D/D/1 recursion
    T_R(k) = max(T_R(k-1), t_k) + tau."""
    rng = np.random.default_rng(0)
    tau = 0.004
    s = sched.Fig10([(sched.TABLE, False, (math.inf, 0.0, 1.0, tau, 0, 1, 0))], math.inf)
    prev = 0.0
    t = 0.0
    for _ in range(500):
        t += float(rng.exponential(0.004))
        p, _, tr, _, est = s.submit(t, -1.0, 0.7, 0.0)
        want = max(prev, t) + tau
        assert p == 0 and est == tau and abs(tr - want) < 1e-12
        prev = want


def test_step5_closed_form_without_deadline_pressure():
    """T_C = inf puts every partition in P_BD, so the choice depends only on the query:
    CPU iff T_CPU < the fastest GPU partition's T, else the first GPU partition in order."""
    rng = np.random.default_rng(1)
    s = sched.Fig10(paper_partitions(), math.inf)
    t = 0.0
    for _ in range(2000):
        t += float(rng.exponential(0.01))
        mb = float(10 ** rng.uniform(0, 4.5))
        cf = float(rng.uniform(0.05, 1.0))
        p, tr, _, _, _ = s.submit(t, mb, cf, float(rng.choice([0.0, 1e-4])))
        t_cpu = 6e-5 * mb ** 0.984 if mb < 512 else 4e-5 * mb + 0.0146
        t_g4 = 0.0008 * cf + 0.0065
        assert p == (0 if t_cpu < t_g4 else 1)


def test_step6_earliest_response_when_nothing_meets_the_deadline():
    """T_C = 0: P_BD is always empty, so every query goes to the partition that answers first
    (greedy earliest-finish list scheduling, written here from its definition)."""
    rng = np.random.default_rng(2)
    parts = paper_partitions()
    s = sched.Fig10(parts, 0.0)
    free = [0.0] * len(parts)
    t = 0.0
    for _ in range(1000):
        t += float(rng.exponential(0.002))
        mb = float(10 ** rng.uniform(0, 3))
        cf = float(rng.uniform(0.05, 1.0))
        finish = []
        for k, (kind, _, fn) in enumerate(parts):
            if kind == sched.CUBE:
                tp = 6e-5 * mb ** 0.984 if mb < 512 else 4e-5 * mb + 0.0146
            else:
                tp = fn[1] * cf + fn[3]
            finish.append(max(free[k], t) + tp)
        best = int(np.argmin(finish))
        p, _, tr, _, _ = s.submit(t, mb, cf, 0.0)
        assert p == best and abs(tr - finish[best]) < 1e-12
        free[best] = finish[best]


def test_translation_queue_serialises_text_queries():
    """Text queries sent to GPU partitions pass through the one translation queue, so their
    translations finish at t_k' = max(t_k'-1, T_O) + T_TRANS; a GPU answer never precedes it."""
    parts = [(sched.TABLE, True, (math.inf, 0.0, 1.0, 0.001, 0, 1, 0))] * 4
    s = sched.Fig10(parts, math.inf)
    tq = 0.0
    for k in range(50):
        t = k * 0.0001
        p, tr, r, _, _ = s.submit(t, -1.0, 1.0, 0.0005)
        tq = max(tq, t) + 0.0005
        assert tr == 1 and r >= tq + 0.001 - 1e-12


def test_unanswerable_query():
    s = sched.Fig10([(sched.CUBE, False, EQ10)], 1.0)
    assert s.submit(0.0, -1.0, 0.5, 0.0)[0] == -1
