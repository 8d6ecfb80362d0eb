"""Pins of the fact-table query oracle (Q_D, Eq. 11-12) against numpy
boolean-mask brute force (library primitives) and against an independent path: the SUM /
fact COUNT of a cube built from the same rows with np.add.at.  CPU only."""
import numpy as np

import oracle
import synth


def _table(nrows, rng):
    dims = [rng.integers(0, n, size=nrows).astype(np.int32) for n in (40, 7, 13, 5)]
    qty = rng.integers(-50, 100, size=nrows).astype(np.int32)
    paid = rng.integers(0, 1 << 14, size=nrows).astype(np.float32)   # integer-valued: exact sums
    return dims + [qty, paid]


def _random_queries(rng, nq, extents):
    qs = []
    for _ in range(nq):
        conds = []
        for c, n in enumerate(extents):
            if rng.random() < 0.6:
                a, b = sorted(rng.integers(-2, n + 2, size=2))
                if rng.random() < 0.05:
                    a, b = b + 1, a            # empty range
                conds.append((c, int(a), int(b)))
        qs.append((conds, int(rng.integers(4, 6)), int(rng.integers(0, 5))))
    return qs


def test_tablescan_vs_numpy_brute_force():
    rng = np.random.default_rng(3)
    cols = _table(5000, rng)
    qs = _random_queries(rng, 400, (40, 7, 13, 5))
    got = oracle.tablescan(cols, qs)
    for q, (conds, dc, op) in enumerate(qs):
        m = np.ones(len(cols[0]), bool)
        for c, lo, hi in conds:
            m &= (cols[c] >= lo) & (cols[c] <= hi)
        vals = cols[dc][m]
        if vals.size == 0:
            assert got["flags"][q] == oracle.RESULT_EMPTY and got["i"][q] == 0 and got["d"][q] == 0
            continue
        assert got["flags"][q] == 0
        isf = cols[dc].dtype == np.float32
        s = vals.astype(np.float64).sum() if isf else int(vals.astype(np.int64).sum())
        want = {oracle.SUM: s, oracle.COUNT: vals.size, oracle.MIN: vals.min(), oracle.MAX: vals.max(),
                oracle.AVG: float(s) / vals.size}[op]
        if op == oracle.COUNT:
            assert got["i"][q] == want
        elif op == oracle.AVG or isf:
            assert got["d"][q] == float(want)
        else:
            assert got["i"][q] == int(want)
    # OpenMP over queries gives identical answers
    assert np.array_equal(oracle.tablescan(cols, qs, nthreads=4), got)


def test_tablescan_equals_cube_path():
    """Independent path: the same rows built into a cube (np.add.at), queried as boxes."""
    rng = np.random.default_rng(4)
    cols = _table(20000, rng)
    ext = (40, 7, 13, 5)
    cube = np.zeros(ext, np.int64)
    np.add.at(cube, tuple(cols[:4]), cols[4].astype(np.int64))
    cnt = np.zeros(ext, np.int64)
    np.add.at(cnt, tuple(cols[:4]), 1)
    boxes = synth.random_boxes(ext, 300, rng)
    qs_sum = [([(d, int(boxes[i, d, 0]), int(boxes[i, d, 1])) for d in range(4)], 4, oracle.SUM) for i in range(300)]
    qs_cnt = [(c, 4, oracle.COUNT) for c, _, _ in qs_sum]
    ts = oracle.tablescan(cols, qs_sum)
    tc = oracle.tablescan(cols, qs_cnt)
    rs = oracle.query(ext, boxes, np.full(300, oracle.SUM, np.int32), cube.astype(np.int32).ravel())
    rc = oracle.query(ext, boxes, np.full(300, oracle.SUM, np.int32), cnt.astype(np.int32).ravel())
    nonempty = tc["flags"] == 0
    assert np.array_equal(ts["i"][nonempty], rs["i"][nonempty])
    assert np.array_equal(tc["i"][nonempty], rc["i"][nonempty])
    assert (rc["i"][~nonempty] == 0).all()
