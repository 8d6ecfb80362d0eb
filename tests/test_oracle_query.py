"""Pins of the oracle's sub-cube query (Eq. 1, Eq. 3) against
things other than itself: a hand-worked example, numpy slicing (brute force that
reduces to library routines), a summed-area-table algorithm (independent),
the affine closed form (any size), and invariants.  CPU only."""
import os

import numpy as np
import pytest

import oracle
import synth

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _load_hand_example():
    rows = []
    with open(os.path.join(GOLDEN, "hand_example_4x4x4.txt")) as f:
        for line in f:
            line = line.split("#", 1)[0].strip()
            if line:
                rows.append(line.split())
    ext = [int(v) for v in rows[0]]
    box = [[int(v) for v in r] for r in rows[1:1 + len(ext)]]
    exp = rows[1 + len(ext)]
    return ext, box, (int(exp[0]), int(exp[1]), int(exp[2]), int(exp[3]), float(exp[4]))


def test_hand_example_fig2():
    ext, box, (cnt, s, mn, mx, avg) = _load_hand_example()
    cells = np.arange(int(np.prod(ext)), dtype=np.int32)         # v = 16x + 4y + z
    ops = [oracle.COUNT, oracle.SUM, oracle.MIN, oracle.MAX, oracle.AVG]
    r = oracle.query(ext, np.array([box] * 5), ops, cells)
    assert list(r["i"][:4]) == [cnt, s, mn, mx]
    assert r["d"][4] == avg
    assert not r["flags"].any()
    # the float32 cube gives the same numbers in d
    rf = oracle.query(ext, np.array([box] * 5), ops, cells.astype(np.float32))
    assert rf["i"][0] == cnt
    assert list(rf["d"][1:]) == [s, mn, mx, avg]


def _numpy_answer(cube, box, op):
    sl = tuple(slice(lo, hi + 1) for lo, hi in box)
    sub = cube[sl]
    if op == oracle.COUNT:
        return sub.size
    if op == oracle.SUM:
        return int(sub.astype(np.int64).sum()) if cube.dtype == np.int32 else float(sub.astype(np.float64).sum())
    if op == oracle.MIN:
        return sub.min()
    if op == oracle.MAX:
        return sub.max()
    s = sub.astype(np.int64).sum() if cube.dtype == np.int32 else sub.astype(np.float64).sum()
    return float(s) / float(sub.size)


@pytest.mark.parametrize("dtype", [np.int32, np.float32])
def test_brute_force_numpy_slicing(dtype):
    """>= 10^4 random boxes over 1-6 dims, extents 1-9 (incl. extent-1 and full dims)."""
    rng = np.random.default_rng(1234 if dtype == np.int32 else 4321)
    total = 0
    for trial in range(60):
        nd = int(rng.integers(1, 7))
        ext = tuple(int(v) for v in rng.integers(1, 10, size=nd))
        n = int(np.prod(ext))
        if dtype == np.int32:
            cells = rng.integers(-(2 ** 31), 2 ** 31, size=n, dtype=np.int64).astype(np.int32)
        else:
            # integer-valued floats below 2^24: fp64 sums are exact in any order
            cells = rng.integers(-(2 ** 20), 2 ** 20, size=n).astype(np.float32)
        cube = cells.reshape(ext)
        nq = 200
        boxes = synth.random_boxes(ext, nq, rng)
        # force some full dims and some extent-1 boxes
        boxes[::7, :, 0] = 0
        boxes[::7, :, 1] = np.array(ext) - 1
        boxes[3::11, 0, 1] = boxes[3::11, 0, 0]
        ops = rng.integers(0, 5, size=nq).astype(np.int32)
        res = oracle.query(ext, boxes, ops, cells)
        for q in range(nq):
            exp = _numpy_answer(cube, boxes[q], ops[q])
            op = ops[q]
            if op == oracle.COUNT:
                assert res["i"][q] == exp
            elif op == oracle.AVG:
                assert res["d"][q] == exp
            elif dtype == np.int32:
                assert res["i"][q] == int(exp)
            else:
                assert res["d"][q] == float(exp)
        total += nq
    assert total >= 10_000


def test_summed_area_table_int_sum():
    """Independent algorithm: N-D prefix sums with 2^N-term inclusion-exclusion."""
    rng = np.random.default_rng(7)
    ext = (6, 5, 4, 7)
    cells = rng.integers(-(2 ** 31), 2 ** 31, size=int(np.prod(ext)), dtype=np.int64).astype(np.int32)
    cube = cells.reshape(ext).astype(object)                       # exact Python ints
    sat = np.zeros(tuple(e + 1 for e in ext), dtype=object)
    sat[1:, 1:, 1:, 1:] = cube
    for ax in range(4):
        sat = np.cumsum(sat, axis=ax)
    boxes = synth.random_boxes(ext, 500, rng)
    res = oracle.query(ext, boxes, np.full(500, oracle.SUM, np.int32), cells)
    nd = len(ext)
    for q in range(500):
        tot = 0
        for corner in range(1 << nd):
            idx, sign = [], 1
            for d in range(nd):
                if corner >> d & 1:
                    idx.append(boxes[q, d, 0])
                    sign = -sign
                else:
                    idx.append(boxes[q, d, 1] + 1)
            tot += sign * sat[tuple(idx)]
        assert res["i"][q] == tot


def _affine_closed_form(box, params):
    """SUM = V*c0 + sum_d c_d*(V/l_d)*(f_d+t_d)*l_d/2; MIN/MAX at corners; AVG = center value."""
    ell = [hi - lo + 1 for lo, hi in box]
    V = 1
    for l in ell:
        V *= l
    s = V * params[0]
    for d, (lo, hi) in enumerate(box):
        s += params[1 + d] * (V // ell[d]) * ((lo + hi) * ell[d] // 2)
    mn = params[0] + sum(params[1 + d] * (lo if params[1 + d] >= 0 else hi) for d, (lo, hi) in enumerate(box))
    mx = params[0] + sum(params[1 + d] * (hi if params[1 + d] >= 0 else lo) for d, (lo, hi) in enumerate(box))
    return V, s, mn, mx


@pytest.mark.parametrize("dtype", [np.int32, np.float32])
def test_affine_closed_form_procedural(dtype):
    """Closed form at sizes far beyond what is materialised (procedural cells)."""
    rng = np.random.default_rng(99)
    ext = (40, 33, 57)
    params = [3, 5, -2, 7]
    boxes = synth.fraction_boxes(ext, 120, rng, 1e-4)
    for op in (oracle.SUM, oracle.MIN, oracle.MAX, oracle.COUNT, oracle.AVG):
        res = oracle.query(ext, boxes, np.full(len(boxes), op, np.int32), dtype=dtype,
                           gen=oracle.GEN_AFFINE, params=np.array(params, float))
        for q in range(len(boxes)):
            V, s, mn, mx = _affine_closed_form(boxes[q].tolist(), params)
            got_i, got_d = int(res["i"][q]), float(res["d"][q])
            if op == oracle.COUNT:
                assert got_i == V
            elif op == oracle.AVG:
                assert got_d == pytest.approx(s / V, rel=1e-15)
            else:
                want = {oracle.SUM: s, oracle.MIN: mn, oracle.MAX: mx}[op]
                assert (got_i if dtype == np.int32 else got_d) == want
    # one full-size 6-D check: every dim full -> the sum of all cells
    ext6 = (16, 16, 16, 16, 16, 4)
    p6 = [1, 1, 2, 3, 4, 5, 6]
    box = [[0, n - 1] for n in ext6]
    res = oracle.query(ext6, np.array([box]), [oracle.SUM], dtype=dtype, gen=oracle.GEN_AFFINE,
                       params=np.array(p6, float))
    V, s, _, _ = _affine_closed_form(box, p6)
    assert (res["i"][0] if dtype == np.int32 else res["d"][0]) == s


def test_generators_agree():
    """The oracle's splitmix64 generator equals synth's numpy one (same published formula)."""
    for dtype in (np.int32, np.float32):
        ext = (7, 9, 11)
        a = oracle.fill(ext, dtype, oracle.GEN_UNIFORM, seed=0x5EED0001)
        b = synth.uniform_cells(int(np.prod(ext)), dtype, 0x5EED0001)
        assert np.array_equal(a, b)
        part = oracle.fill(ext, dtype, oracle.GEN_UNIFORM, seed=0x5EED0001, first=100, count=50)
        assert np.array_equal(part, b[100:150])
    # reference value of splitmix64 (Vigna's published sequence for state 0: first output)
    assert oracle.splitmix64(0, 0) == 0xE220A8397B1DCDAF
    assert int(synth.splitmix64(0, [0])[0]) == 0xE220A8397B1DCDAF
    ext = (5, 6)
    p = [1.0, 2.0, -3.0]
    assert np.array_equal(oracle.fill(ext, np.int32, oracle.GEN_AFFINE, params=p),
                          synth.affine_cells(ext, np.int32, p))
    # procedural query == materialised query
    cells = synth.uniform_cells(7 * 9 * 11, np.float32, 5)
    rng = np.random.default_rng(3)
    boxes = synth.random_boxes((7, 9, 11), 100, rng)
    ops = synth.ops_uniform(100, rng)
    r1 = oracle.query((7, 9, 11), boxes, ops, cells)
    r2 = oracle.query((7, 9, 11), boxes, ops, dtype=np.float32, gen=oracle.GEN_UNIFORM, seed=5)
    assert np.array_equal(r1, r2)


def test_invariants():
    rng = np.random.default_rng(11)
    ext = (9, 8, 7, 6)
    for dtype in (np.int32, np.float32):
        cells = synth.uniform_cells(int(np.prod(ext)), dtype, 77)
        full = [[0, n - 1] for n in ext]
        # full-cube query equals the sum of all cells
        r = oracle.query(ext, np.array([full]), [oracle.SUM], cells)
        tot = int(cells.astype(np.int64).sum()) if dtype == np.int32 else float(cells.astype(np.float64).sum())
        got = r["i"][0] if dtype == np.int32 else r["d"][0]
        if dtype == np.int32:
            assert got == tot
        else:
            assert got == pytest.approx(tot, rel=1e-12)
        # splitting a box along any dim at any cut: SUM/COUNT add, MIN/MAX combine
        boxes = synth.random_boxes(ext, 200, rng)
        for q in range(200):
            b = boxes[q]
            d = int(rng.integers(0, 4))
            if b[d, 0] == b[d, 1]:
                continue
            cut = int(rng.integers(b[d, 0], b[d, 1]))
            b1, b2 = b.copy(), b.copy()
            b1[d, 1] = cut
            b2[d, 0] = cut + 1
            trio = np.stack([b, b1, b2])
            res = {op: oracle.query(ext, trio, [op] * 3, cells) for op in range(5)}
            f = "i" if dtype == np.int32 else "d"
            assert res[oracle.COUNT]["i"][0] == res[oracle.COUNT]["i"][1] + res[oracle.COUNT]["i"][2]
            if dtype == np.int32:
                assert res[oracle.SUM]["i"][0] == res[oracle.SUM]["i"][1] + res[oracle.SUM]["i"][2]
            else:
                assert res[oracle.SUM]["d"][0] == pytest.approx(res[oracle.SUM]["d"][1] + res[oracle.SUM]["d"][2],
                                                                rel=1e-12)
            assert res[oracle.MIN][f][0] == min(res[oracle.MIN][f][1], res[oracle.MIN][f][2])
            assert res[oracle.MAX][f][0] == max(res[oracle.MAX][f][1], res[oracle.MAX][f][2])
            assert res[oracle.MIN][f][0] <= res[oracle.AVG]["d"][0] <= res[oracle.MAX][f][0]
        # order invariance and batch splitting
        ops = synth.ops_uniform(200, rng)
        r_all = oracle.query(ext, boxes, ops, cells)
        perm = rng.permutation(200)
        r_perm = oracle.query(ext, boxes[perm], ops[perm], cells)
        assert np.array_equal(r_all[perm], r_perm)
        r_a = oracle.query(ext, boxes[:77], ops[:77], cells)
        assert np.array_equal(r_all[:77], r_a)
        # OpenMP loop over queries gives identical answers
        r_omp = oracle.query(ext, boxes, ops, cells, nthreads=4)
        assert np.array_equal(r_all, r_omp)


def test_empty_and_bounds():
    ext = (4, 5)
    cells = np.arange(20, dtype=np.int32)
    boxes = np.array([[[2, 1], [0, 4]], [[0, 3], [3, 3]]])
    r = oracle.query(ext, boxes, [oracle.SUM, oracle.COUNT], cells)
    assert r["flags"][0] == oracle.RESULT_EMPTY and r["i"][0] == 0 and r["d"][0] == 0
    assert r["flags"][1] == 0 and r["i"][1] == 4
    for op in range(5):
        r = oracle.query(ext, boxes[:1], [op], cells)
        assert r["flags"][0] == oracle.RESULT_EMPTY
    with pytest.raises(IndexError):
        oracle.query(ext, np.array([[[0, 4], [0, 4]]]), [oracle.SUM], cells)
    with pytest.raises(IndexError):
        oracle.query(ext, np.array([[[-1, 2], [0, 4]]]), [oracle.SUM], cells)
    # a 1-D, 1-cell cube
    r = oracle.query((1,), np.array([[[0, 0]]]), [oracle.MAX], np.array([-5], np.int32))
    assert r["i"][0] == -5
