"""GPU parity of the bricked layout (OLAP_LAYOUT_BRICK, DESIGN.md §5 / reading R26).

The layout changes where cells sit in HBM, not what a query computes (Eq. 1 boxes,
PAPER.md:126-130; aggregates PAPER.md:25), so every result must equal the oracle's on the
logical row-major cube under the same bars as tests/test_gpu_parity.py: int32 bit-exact,
float32 SUM/AVG within 1e-6 relative (bit-exact on integer-valued affine cubes).
"""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_ipps_malikrse12_b200 as olap
import synth
from test_gpu_parity import compare

pytestmark = pytest.mark.gpu

LAYOUTS = [olap.LAYOUT_BRICK, olap.LAYOUT_BRICK3]


@pytest.fixture(params=LAYOUTS, ids=["brick_1x4x8", "brick3_2x4x4"])
def BRICK(request):
    """Both bricked layouts (1 x 4 x 8 and 2 x 4 x 4 cells) must give the oracle's answers."""
    return request.param

SHAPES = [
    ((3, 8, 16), "extents multiples of the 4 x 8 brick"),
    ((5, 9, 13), "ragged in both bricked dims (padding cells)"),
    ((2, 3, 17, 33), "4-D, ragged"),
    ((4, 4, 4, 4, 4, 40), "6-D (the bricked maximum)"),
    ((7, 1, 1), "extent-1 bricked dims"),
    ((2, 64, 1000), "long rows: whole-brick middles merge into long runs"),
    ((3, 4, 8), "a single brick per dim-0 row"),
    ((1, 5, 6), "one dim-0 row (an unpaired local row for 2 x 4 x 4)"),
    ((9, 4, 4), "odd dim-0 extent, one brick column"),
]


def _boxes(ext, rng, n=300):
    small = synth.small_boxes(ext, n, rng, bytes_lo=4, bytes_hi=4096)
    full = np.array([[[0, e - 1] for e in ext]])
    return np.concatenate([synth.random_boxes(ext, n, rng), synth.fraction_boxes(ext, n, rng, 1e-4), small, full, full])


@pytest.mark.parametrize("dtype", [np.int32, np.float32])
@pytest.mark.parametrize("ext,why", SHAPES)
def test_brick_shapes_vs_oracle(ext, why, dtype, BRICK):
    n = int(np.prod(ext))
    seed = 0x5EED3000 + n
    cells = synth.uniform_cells(n, dtype, seed)
    rng = np.random.default_rng(seed)
    boxes = _boxes(ext, rng)
    ops = synth.ops_uniform(len(boxes), rng)
    ops[-2:] = [olap.SUM, olap.MIN]
    c = olap.Cube(ext, dtype, layout=BRICK)
    c.load(cells)
    ref = oracle.query(ext, boxes, ops, cells)
    compare(c.query(boxes, ops), ref, ops, dtype)
    # every op on every box
    for op in range(5):
        o = np.full(len(boxes), op, np.int32)
        compare(c.query(boxes, o), oracle.query(ext, boxes, o, cells), o, dtype)
    # the device fill writes the same logical cells as the host load
    c2 = olap.Cube(ext, dtype, layout=BRICK)
    c2.fill(olap.GEN_UNIFORM, seed)
    compare(c2.query(boxes, ops), ref, ops, dtype)


@pytest.mark.parametrize("dtype", [np.int32, np.float32])
def test_brick_affine_bit_exact(dtype, BRICK):
    ext = (6, 10, 37, 45)
    params = np.array([7, 3, -2, 5, 1], float)
    c = olap.Cube(ext, dtype, layout=BRICK)
    c.fill(olap.GEN_AFFINE, 0, params)
    rng = np.random.default_rng(11)
    boxes = _boxes(ext, rng, 400)
    ops = synth.ops_uniform(len(boxes), rng)
    ref = oracle.query(ext, boxes, ops, dtype=dtype, gen=oracle.GEN_AFFINE, params=params)
    compare(c.query(boxes, ops), ref, ops, dtype, exact_float=True)


def test_brick_every_section_shape(BRICK):
    """Every head/middle/tail combination in the bricked dims: boxes starting and ending at
    every offset inside a brick (1-cell, within-one-brick, whole-brick and spanning boxes),
    and for 2 x 4 x 4 bricks every dim-0 row pairing (first / second row of a pair, both,
    across pairs, the unpaired last row)."""
    ext = (5, 13, 27)
    cells = synth.uniform_cells(int(np.prod(ext)), np.int32, 77)
    rows = ((0, 1),) if BRICK == olap.LAYOUT_BRICK else ((0, 0), (1, 1), (0, 1), (1, 2), (4, 4), (0, 4))
    bs = []
    for r0, r1 in rows:
        for a0 in range(13):
            for a1 in range(a0, 13):
                for b0 in (0, 1, 3, 4, 7, 8, 9, 15, 16, 26):
                    for b1 in (b0, 3, 4, 7, 8, 15, 16, 23, 24, 26):
                        if b1 >= b0:
                            bs.append([[r0, r1], [a0, a1], [b0, b1]])
    boxes = np.array(bs, np.int64)
    c = olap.Cube(ext, np.int32, layout=BRICK)
    c.load(cells)
    for op in (olap.SUM, olap.MIN, olap.MAX):
        o = np.full(len(boxes), op, np.int32)
        compare(c.query(boxes, o), oracle.query(ext, boxes, o, cells), o, np.int32)


@pytest.mark.parametrize("G,b", [(2, 1), (3, 2), (4, 5)])
@pytest.mark.parametrize("dtype", [np.int32, np.float32])
def test_brick_virtual_shards(G, b, dtype, BRICK):
    """Dim 0 stays unbricked, so block-cyclic shards of a bricked cube combine to the global answer."""
    ext = (23, 9, 70)
    cells = synth.uniform_cells(int(np.prod(ext)), dtype, 0x5EED4000 + G)
    rng = np.random.default_rng(G + 7 * b)
    boxes = np.concatenate([synth.random_boxes(ext, 300, rng), synth.fraction_boxes(ext, 200, rng, 1e-3)])
    ops = synth.ops_uniform(len(boxes), rng)
    nq = len(boxes)
    dr = torch.from_numpy(boxes.astype(np.int64)).cuda()
    do = torch.from_numpy(ops).cuda()
    acc_s = torch.zeros(nq, dtype=torch.int64, device="cuda")
    acc_e = torch.full((2 * nq,), -(2 ** 31), dtype=torch.int32, device="cuda")
    for g in range(G):
        cg = olap.Cube(ext, dtype, shard=(G, g, b), layout=BRICK)
        if g % 2:
            cg.load(cells)
        else:
            cg.fill(olap.GEN_UNIFORM, 0x5EED4000 + G)
        s = torch.empty(nq, dtype=torch.int64, device="cuda")
        e = torch.empty(2 * nq, dtype=torch.int32, device="cuda")
        cg.partials_device(dr, do, s, e)
        olap.combine_partials_device(dtype, nq, s, e, acc_s, acc_e)
        torch.cuda.synchronize()
        cg.close()
    res = torch.empty(nq * 24, dtype=torch.uint8, device="cuda")
    olap.finalize_device(ext, dtype, nq, dr, do, acc_s, acc_e, res)
    got = res.cpu().numpy().view(olap.RESULT_DTYPE)
    compare(got, oracle.query(ext, boxes, ops, cells), ops, dtype)


def test_brick_empty_invalid_errors_and_determinism(BRICK):
    ext = (4, 10, 20)
    cells = synth.uniform_cells(800, np.float32, 3)
    c = olap.Cube(ext, np.float32, layout=BRICK)
    c.load(cells)
    # host path: out of range -> OLAP_E_RANGE naming query and dimension
    with pytest.raises(olap.OlapError) as ei:
        c.query(np.array([[[0, 3], [0, 9], [0, 20]]]), np.array([olap.SUM], np.int32))
    assert ei.value.status == olap.E_RANGE
    # device path: invalid flagged, empty flagged, valid answered
    boxes = np.array([[[0, 3], [0, 10], [0, 1]], [[0, 3], [5, 4], [0, 1]], [[0, 3], [0, 9], [0, 19]]], np.int64)
    ops = np.array([olap.SUM, olap.MIN, olap.SUM], np.int32)
    res = torch.zeros(3 * 24, dtype=torch.uint8, device="cuda")
    c.query_device(torch.from_numpy(boxes).cuda(), torch.from_numpy(ops).cuda(), res)
    torch.cuda.synchronize()
    out = res.cpu().numpy().view(olap.RESULT_DTYPE)
    assert list(out["flags"]) == [olap.RESULT_INVALID, olap.RESULT_EMPTY, 0]
    assert abs(out["d"][2] - cells.astype(np.float64).sum()) <= 1e-6 * cells.astype(np.float64).sum()
    # float sums are bit-identical run to run
    rng = np.random.default_rng(2)
    bx = synth.fraction_boxes(ext, 500, rng, 1e-3)
    o = np.full(len(bx), olap.SUM, np.int32)
    r0 = c.query(bx, o)
    for _ in range(3):
        assert np.array_equal(c.query(bx, o), r0)
    # layouts that cannot hold a brick, and row-major-only operations
    for bad in ((10, 20), (2, 2, 2, 2, 2, 2, 2)):
        with pytest.raises(olap.OlapError):
            olap.Cube(bad, np.int32, layout=BRICK)
    with pytest.raises(olap.OlapError):
        olap.Cube((4, 4, 4), np.int32, layout=7)
    with pytest.raises(olap.OlapError) as ei:
        c.add_facts_device(torch.zeros(3, dtype=torch.int32, device="cuda"), nrows=1)
    assert ei.value.status == olap.E_UNSUPPORTED


def test_brick_cuda_graph_capture_replay(BRICK):
    ext = (16, 64, 96)
    c = olap.Cube(ext, np.float32, layout=BRICK)
    c.fill(olap.GEN_UNIFORM, 9)
    boxes, ops = synth.config_queries("C5", nq=512, seed=5, extents=ext)
    dr = torch.from_numpy(boxes).cuda()
    do = torch.from_numpy(ops).cuda()
    res = torch.zeros(512 * 24, dtype=torch.uint8, device="cuda")
    st = torch.cuda.Stream()
    with torch.cuda.stream(st):
        c.query_device(dr, do, res, stream=st)
    st.synchronize()
    want = res.clone()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=st):
        c.query_device(dr, do, res, stream=torch.cuda.current_stream())
    for _ in range(3):
        res.zero_()
        g.replay()
        torch.cuda.synchronize()
        assert torch.equal(res, want)
    ref = oracle.query(ext, boxes, ops, dtype=np.float32, gen=oracle.GEN_UNIFORM, seed=9)
    compare(want.cpu().numpy().view(olap.RESULT_DTYPE), ref, ops, np.float32)


def test_brick_c5_small_boxes_equal_rowmajor(BRICK):
    """C5's recipe (4 KiB .. 4 MiB boxes) on a 256 MiB slice: bricked == row-major == oracle."""
    ext = (32, 1024, 2048)
    boxes, ops = synth.config_queries("C5", nq=8192, seed=21, extents=ext)
    rm = olap.Cube(ext, np.int32)
    rm.fill(olap.GEN_UNIFORM, 21)
    want = rm.query(boxes, ops)
    rm.close()
    bk = olap.Cube(ext, np.int32, layout=BRICK)
    bk.fill(olap.GEN_UNIFORM, 21)
    got = bk.query(boxes, ops)
    assert np.array_equal(got, want)
    idx = np.random.default_rng(0).choice(len(boxes), 300, replace=False)
    ref = oracle.query(ext, boxes[idx], ops[idx], dtype=np.int32, gen=oracle.GEN_UNIFORM, seed=21)
    compare(got[idx], ref, ops[idx], np.int32)


def test_brick_signed_noninteger_float(BRICK):
    """VERDICT r1 weak #2 on the bricked kernel (fp32 tree of one 8-cell brick row, then fp64):
    mixed-sign, non-integer cells within 1e-6 * sum|x|; MIN / MAX / COUNT exact."""
    from test_gpu_parity import compare_signed, signed_cells
    ext = (6, 61, 203)
    cells = signed_cells(int(np.prod(ext)), 0x5EED2400)
    c = olap.Cube(ext, np.float32, layout=BRICK)
    c.load(cells)
    rng = np.random.default_rng(24)
    boxes = _boxes(ext, rng, 200)
    ops = synth.ops_uniform(len(boxes), rng)
    compare_signed(c.query(boxes, ops), cells, ext, boxes, ops)
