"""Pins of oracle.factbuild (oracle_factbuild, the cube built from fact rows, PAPER.md:101;
reading R27): against numpy's unbuffered np.add.at (a library primitive) -- int32 wrapping
mod 2^32, float32 accumulated per cell in fp64 in row order and rounded once -- plus the
count cube (bincount) and rows with out-of-range ids.  CPU only."""
import numpy as np

import oracle


def _rows(ext, nrows, rng):
    return np.stack([rng.integers(0, n, size=nrows) for n in ext]).astype(np.int32)


def test_int32_build_wraps_like_add_at():
    rng = np.random.default_rng(1)
    ext = (5, 4, 3)
    ids = _rows(ext, 20_000, rng)
    vals = rng.integers(-2 ** 31, 2 ** 31 - 1, size=20_000, dtype=np.int64).astype(np.int32)
    init = rng.integers(-1000, 1000, size=ext).astype(np.int32)
    acc = init.astype(np.int64).copy()
    np.add.at(acc, tuple(ids), vals.astype(np.int64))
    want = (acc & 0xFFFFFFFF).astype(np.uint32).view(np.int32).reshape(-1)
    assert np.array_equal(oracle.factbuild(ext, ids, vals, init), want)
    # count cube: +1 per row
    cnt = oracle.factbuild(ext, ids, None, np.zeros(ext, np.int32))
    assert np.array_equal(cnt, np.bincount(np.ravel_multi_index(tuple(ids), ext), minlength=60))


def test_float32_build_fp64_row_order_one_rounding():
    rng = np.random.default_rng(2)
    ext = (6, 7, 5)
    ids = _rows(ext, 30_000, rng)
    vals = (rng.standard_normal(30_000) * rng.choice([1e-2, 1.0, 1e4], size=30_000)).astype(np.float32)
    init = rng.standard_normal(ext).astype(np.float32)
    acc = np.zeros(ext, np.float64)
    np.add.at(acc, tuple(ids), vals.astype(np.float64))
    want = (init.astype(np.float64) + acc).astype(np.float32).reshape(-1)
    got = oracle.factbuild(ext, ids, vals, init)
    assert np.array_equal(got, want)
    # fp32 accumulation or rounding at every add would differ (the pin sees those mistakes)
    acc32 = init.copy()
    np.add.at(acc32, tuple(ids), vals)
    assert not np.array_equal(got, acc32.reshape(-1))


def test_out_of_range_ids_add_nothing():
    ext = (3, 3)
    ids = np.array([[0, 3, -1, 2], [1, 1, 0, 5]], np.int32)
    got = oracle.factbuild(ext, ids, np.array([1.5, 2.0, 4.0, 8.0], np.float32), np.zeros(ext, np.float32))
    want = np.zeros(9, np.float32)
    want[1] = 1.5
    assert np.array_equal(got, want)
