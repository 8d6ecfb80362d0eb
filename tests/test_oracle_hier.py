"""Pins of the multi-resolution cube-set oracle (Fig. 1, Eq. 1-2):
roll-up vs numpy np.add.at / np.minimum.at over the level maps (library primitives),
SUM preserved across levels (invariant), range conversion vs a direct definition on the
date hierarchy (year/month/day).  CPU only."""
import datetime as dt

import numpy as np

import oracle
import synth


def test_rollup_vs_numpy_ufunc_at():
    rng = np.random.default_rng(5)
    hier = [synth.random_hierarchy(n, 3, rng) for n in (9, 7, 11)]
    fine = rng.integers(-1000, 1000, size=(9, 7, 11)).astype(np.int32)
    for rc in (0, 1):
        ext_c = tuple(int(h[rc].max()) + 1 for h in hier)
        idx = np.ix_(*[h[rc] for h in hier])
        for op, ufunc, init in ((oracle.SUM, np.add, 0), (oracle.MIN, np.minimum, 2 ** 31 - 1),
                                (oracle.MAX, np.maximum, -2 ** 31)):
            want = np.full(ext_c, init, np.int64)
            grid = np.meshgrid(*[h[rc] for h in hier], indexing="ij")
            ufunc.at(want, tuple(g.ravel() for g in grid), fine.astype(np.int64).ravel())
            got = oracle.rollup(hier, fine, 2, rc, op)
            assert np.array_equal(got.astype(np.int64), want)
        # SUM is preserved across levels (roll-up of a roll-up == direct roll-up)
        assert oracle.rollup(hier, fine, 2, rc).astype(np.int64).sum() == fine.astype(np.int64).sum()
    mid = oracle.rollup(hier, fine, 2, 1)
    assert np.array_equal(oracle.rollup(hier, mid, 1, 0), oracle.rollup(hier, fine, 2, 0))


def test_convert_range_on_dates():
    ids = synth.date_hierarchy()
    d0 = dt.date(1998, 1, 1)
    # months [1999-03, 2000-02] (level 1) -> days
    lo, hi = oracle.convert_range(ids, 1, 2, 14, 25)
    assert (d0 + dt.timedelta(lo)).isoformat() == "1999-03-01"
    assert (d0 + dt.timedelta(hi)).isoformat() == "2000-02-29"
    # year 2000 -> months 24..35
    assert oracle.convert_range(ids, 0, 1, 2, 2) == (24, 35)
    # same level: identity; empty range stays empty
    assert oracle.convert_range(ids, 2, 2, 100, 200) == (100, 200)
    lo, hi = oracle.convert_range(ids, 1, 2, 5, 4)
    assert lo > hi


def test_rollup_float32_vs_numpy_fp64_then_one_rounding():
    """the float32 branch of oracle_rollup.  The definition (R27-like
    reading of PAPER.md:103: a coarse cell aggregates its fine cells) accumulates in fp64 and
    rounds once; numpy's np.add.at into float64 in the same (row-major) order, cast once, must
    agree bit for bit.  Signed non-integer cells with 2^24-scale spread make fp32 accumulation or
    per-add rounding visible."""
    rng = np.random.default_rng(11)
    hier = [synth.random_hierarchy(n, 3, rng) for n in (13, 9, 17)]
    fine = (rng.standard_normal((13, 9, 17)) * rng.choice([1e-3, 1.0, 3e3], size=(13, 9, 17))).astype(np.float32)
    for rc in (0, 1):
        ext_c = tuple(int(h[rc].max()) + 1 for h in hier)
        grid = np.meshgrid(*[h[rc] for h in hier], indexing="ij")
        acc = np.zeros(ext_c, np.float64)
        np.add.at(acc, tuple(g.ravel() for g in grid), fine.astype(np.float64).ravel())
        got = oracle.rollup(hier, fine, 2, rc)
        assert got.dtype == np.float32
        assert np.array_equal(got, acc.astype(np.float32))
        # fp32 accumulation would differ somewhere (the pin can see that mistake)
        acc32 = np.zeros(ext_c, np.float32)
        np.add.at(acc32, tuple(g.ravel() for g in grid), fine.ravel())
        assert not np.array_equal(got, acc32)
        for op, ufunc in ((oracle.MIN, np.minimum), (oracle.MAX, np.maximum)):
            want = np.full(ext_c, np.inf if op == oracle.MIN else -np.inf, np.float32)
            ufunc.at(want, tuple(g.ravel() for g in grid), fine.ravel())
            assert np.array_equal(oracle.rollup(hier, fine, 2, rc, op), want)


def test_rollup_int32_sum_wraps_mod_2_32():
    """int32 SUM roll-up wraps into the int32 cell (two's complement, mod 2^32)."""
    rng = np.random.default_rng(12)
    hier = [synth.random_hierarchy(n, 2, rng) for n in (8, 6)]
    fine = rng.integers(2 ** 30, 2 ** 31 - 1, size=(8, 6)).astype(np.int32)  # sums overflow int32
    ext_c = tuple(int(h[0].max()) + 1 for h in hier)
    grid = np.meshgrid(*[h[0] for h in hier], indexing="ij")
    acc = np.zeros(ext_c, np.int64)
    np.add.at(acc, tuple(g.ravel() for g in grid), fine.astype(np.int64).ravel())
    want = ((acc & 0xFFFFFFFF).astype(np.uint32)).view(np.int32)
    got = oracle.rollup(hier, fine, 1, 0)
    assert (acc > 2 ** 31 - 1).any()
    assert np.array_equal(got, want)
