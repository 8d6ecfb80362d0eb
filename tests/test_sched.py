"""The dispatcher (olap_sched_*, host code in the product library) against oracle.sched
(Fig. 10).  CPU only: the scheduler makes no CUDA call."""
import math

import numpy as np
import pytest

import paper_conf_ipps_malikrse12_b200 as olap
from oracle import sched as osched

from test_oracle_sched import load_golden, paper_partitions


def _lib_parts(parts):
    return [(olap.PART_CUBE if k == osched.CUBE else olap.PART_TABLE, nt, fn) for k, nt, fn in parts]


def test_golden_paper_system_through_the_library():
    s = olap.Scheduler(_lib_parts(paper_partitions()), 0.020)
    for ev in load_golden():
        if ev[0] == "C":
            s.complete(ev[1], ev[2], ev[3])
            continue
        _, t, mb, cf, tt, p, tr, r = ev
        d = s.submit([(t, mb, cf, tt)])[0]
        assert (d["partition"], d["translated"]) == (p, tr) and abs(d["t_response"] - r) < 5e-7


def _random_parts(rng):
    parts = []
    for _ in range(int(rng.integers(1, 9))):
        kind = osched.CUBE if rng.random() < 0.3 else osched.TABLE
        if rng.random() < 0.5:   # Eq. 7/10 shape: power law on range A, linear on range B
            fn = (float(rng.choice([64.0, 512.0, math.inf])), float(rng.uniform(1e-5, 1e-4)),
                  float(rng.uniform(0.8, 1.1)), 0.0, float(rng.uniform(1e-5, 1e-4)), 1.0, float(rng.uniform(0, 0.02)))
        else:                    # Eq. 14 / roofline shape: a x + b
            fn = (math.inf, float(rng.uniform(1e-4, 5e-3)), 1.0, float(rng.uniform(1e-4, 3e-2)), 0.0, 1.0, 0.0)
        parts.append((kind, bool(rng.random() < 0.6), fn))
    return parts


@pytest.mark.parametrize("seed", range(12))
def test_random_streams_match_the_oracle(seed):
    rng = np.random.default_rng(seed)
    parts = _random_parts(rng)
    t_c = float(rng.choice([1e-3, 5e-3, 2e-2, 0.1, math.inf]))
    ora = osched.Fig10(parts, t_c)
    lib = olap.Scheduler(_lib_parts(parts), t_c)
    t = 0.0
    outstanding = []
    for k in range(3000):
        t += float(rng.exponential(0.002))
        mb = float(10 ** rng.uniform(-1, 4)) if rng.random() < 0.8 else -1.0
        cf = float(rng.uniform(0.05, 1.0)) if rng.random() < 0.9 else -1.0
        tt = float(rng.uniform(0, 2e-3)) if rng.random() < 0.5 else 0.0
        want = ora.submit(t, mb, cf, tt)
        got = lib.submit([(t, mb, cf, tt)])[0]
        assert got["partition"] == want[0] and got["translated"] == want[1], (k, got, want)
        if want[0] >= 0:
            assert got["t_response"] == want[2] and got["t_deadline"] == want[3] and got["t_est"] == want[4]
            outstanding.append((want[0], want[4]))
        # completions in random order with real times off the estimate
        if outstanding and rng.random() < 0.5:
            p, est = outstanding.pop(int(rng.integers(0, len(outstanding))))
            real = est * float(rng.uniform(0.5, 1.5))
            ora.complete(p, est, real)
            lib.complete(p, est, real)
        if k % 500 == 0:
            q = lib.queues()
            assert list(q[:-1]) == ora.t_q and q[-1] == ora.t_q_trans


def test_batch_submit_equals_one_by_one():
    rng = np.random.default_rng(99)
    parts = _random_parts(rng)
    qs = np.zeros(500, dtype=olap.SCHED_QUERY_DTYPE)
    qs["t_arrival"] = np.cumsum(rng.exponential(0.001, 500))
    qs["cube_mb"] = 10 ** rng.uniform(0, 3, 500)
    qs["col_frac"] = rng.uniform(0.1, 1, 500)
    qs["t_trans"] = rng.uniform(0, 1e-3, 500)
    a = olap.Scheduler(_lib_parts(parts), 0.01).submit(qs)
    s = olap.Scheduler(_lib_parts(parts), 0.01)
    b = np.concatenate([s.submit(qs[i:i + 1]) for i in range(500)])
    assert a.tobytes() == b.tobytes()


def test_deadline_flag_is_consistent():
    """A query placed by step 5 meets its deadline on the estimate; step 6 placements do not."""
    rng = np.random.default_rng(5)
    s = olap.Scheduler(_lib_parts(paper_partitions()), 0.015)
    qs = np.zeros(4000, dtype=olap.SCHED_QUERY_DTYPE)
    qs["t_arrival"] = np.cumsum(rng.exponential(0.0015, 4000))
    qs["cube_mb"] = 10 ** rng.uniform(0, 3.5, 4000)
    qs["col_frac"] = rng.uniform(0.1, 1, 4000)
    d = s.submit(qs)
    met = d["t_response"] < d["t_deadline"]
    assert met.any() and (~met).any()          # the load mixes both regimes
    assert (d["t_response"] >= qs["t_arrival"] + d["t_est"] - 1e-15).all()


def test_errors():
    with pytest.raises(olap.OlapError):
        olap.Scheduler([], 1.0)
    with pytest.raises(olap.OlapError):
        olap.Scheduler([(olap.PART_CUBE, False, olap.perf_fn(1.0))], 0.0)
    with pytest.raises(olap.OlapError):
        olap.Scheduler([(7, False, olap.perf_fn(1.0))], 1.0)
    s = olap.Scheduler([(olap.PART_TABLE, True, olap.perf_fn(1e-3, b1=1e-3))], 1.0)
    with pytest.raises(olap.OlapError):
        s.submit([(0.0, 1.0, float("nan"), 0.0)])
    with pytest.raises(olap.OlapError):
        s.complete(3, 0.0, 0.0)
    d = s.submit([(0.0, 1.0, -1.0, 0.0)])[0]
    assert d["partition"] == -1
