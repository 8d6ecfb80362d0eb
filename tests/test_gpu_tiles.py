"""GPU parity of the tile-shared scan (tiles.cuh) against the oracle.

Cubes larger than 64 MiB get the tile path; the device takes it for batches whose boxes
overlap enough (every staged byte reused >= 4 times).  The shapes below put the tile
dimension kt at different depths, with ragged last chunks, a padded inner pitch, 16-B and
4-B slots, a 1-D cube, int32 and float32 cells.  Bars as in test_gpu_parity.py.
"""
import os

import numpy as np
import pytest

import oracle
import paper_conf_ipps_malikrse12_b200 as olap
import synth
from test_gpu_parity import compare

pytestmark = pytest.mark.gpu

TILE_CELLS_MAX = 16384   # tiles.cuh kTileCellsMax (64 KiB)

TILE_SHAPES = [
    ((40, 16, 20, 16, 160), "kt=2, chunks 7/7/6 (ragged), 32-B slots"),
    ((6, 3000003), "kt = innermost dim: chunks of a padded 3M-cell row"),
    ((17000003,), "1-D: chunks of the only dim"),
    ((1500, 1000, 12), "inner 12: 16-B slots, tile = one dim-0 row"),
    ((4000, 600, 7), "inner 7 padded to 8"),
    ((3, 5, 7, 11, 13, 17, 19, 5), "8-D, odd extents"),
]


def _batch(ext, rng, nq=160):
    big = synth.fraction_boxes(ext, nq, rng, 1e-3, 0.3)
    full = np.array([[[0, e - 1] for e in ext]] * 4)
    boxes = np.concatenate([big, full])
    ops = synth.ops_uniform(len(boxes), rng)
    ops[-4:] = [olap.SUM, olap.MIN, olap.MAX, olap.AVG]
    return boxes, ops


@pytest.mark.parametrize("dtype", [np.int32, np.float32])
@pytest.mark.parametrize("ext,why", TILE_SHAPES)
def test_tile_path_parity(ext, why, dtype):
    if int(np.prod(ext)) * 4 <= (64 << 20):
        ext = ext[:-1] + (ext[-1] * 2,)   # keep every shape above the 64 MiB threshold
    seed = 0x5EED2000 + int(np.prod(ext)) % 1000
    c = olap.Cube(ext, dtype)
    c.fill(olap.GEN_UNIFORM, seed)
    en, tcells, ntiles, _ = c.tile_stats()
    assert en and 0 < tcells <= TILE_CELLS_MAX and ntiles >= 1
    rng = np.random.default_rng(seed)
    boxes, ops = _batch(ext, rng)
    got = c.query(boxes, ops)
    assert c.tile_stats()[3], "batch expected to take the tile path"
    ref = oracle.query(ext, boxes, ops, dtype=dtype, gen=oracle.GEN_UNIFORM, seed=seed,
                       nthreads=oracle.max_threads())
    compare(got, ref, ops, dtype)


@pytest.mark.parametrize("dtype", [np.int32, np.float32])
def test_tile_path_affine_bit_exact(dtype):
    """Integer-valued affine cells: every fp64 partial is exact, so float SUM/AVG are bit-exact."""
    ext = (40, 16, 16, 16, 160)
    params = np.array([3, 1, -2, 5, 1, 2], float)
    c = olap.Cube(ext, dtype)
    c.fill(olap.GEN_AFFINE, 0, params)
    boxes, ops = _batch(ext, np.random.default_rng(9))
    got = c.query(boxes, ops)
    assert c.tile_stats()[3]
    ref = oracle.query(ext, boxes, ops, dtype=dtype, gen=oracle.GEN_AFFINE, params=params,
                       nthreads=oracle.max_threads())
    compare(got, ref, ops, dtype, exact_float=True)


def test_tile_and_item_paths_agree_int():
    """The same int32 batch through the tile path and through the item path (tiles disabled
    for the second cube): bit-identical results."""
    ext = (40, 16, 16, 16, 160)
    a = olap.Cube(ext, np.int32)
    a.fill(olap.GEN_UNIFORM, 5)
    os.environ["OLAP_NO_TILES"] = "1"
    try:
        b = olap.Cube(ext, np.int32)
    finally:
        del os.environ["OLAP_NO_TILES"]
    b.fill(olap.GEN_UNIFORM, 5)
    assert not b.tile_stats()[0]
    boxes, ops = synth.config_queries("C2a", nq=1024, extents=ext)
    ra, rb = a.query(boxes, ops), b.query(boxes, ops)
    assert a.tile_stats()[3]
    assert ra.tobytes() == rb.tobytes()


def test_tile_path_deterministic_and_small_boxes_take_items():
    ext = (32, 16, 16, 16, 256)
    c = olap.Cube(ext, np.float32)
    c.fill(olap.GEN_UNIFORM, 17)
    boxes, ops = synth.config_queries("C2a", nq=2048, extents=ext)
    r = c.query(boxes, ops)
    assert c.tile_stats()[3]
    for _ in range(2):
        assert c.query(boxes, ops).tobytes() == r.tobytes()
    # tiny non-overlapping boxes: staging whole tiles would not pay -> item path, same answers
    rng = np.random.default_rng(3)
    sb = synth.small_boxes(ext, 500, rng, bytes_lo=64, bytes_hi=4096)
    so = synth.ops_uniform(500, rng)
    got = c.query(sb, so)
    assert not c.tile_stats()[3]
    ref = oracle.query(ext, sb, so, dtype=np.float32, gen=oracle.GEN_UNIFORM, seed=17)
    compare(got, ref, so, np.float32)


@pytest.mark.parametrize("G,b", [(2, 1), (3, 2)])
def test_tile_path_on_shards(G, b):
    """Shards (block-cyclic dim 0) each take the tile path on their local box; the combined
    partials equal the unsharded answer."""
    import torch
    ext = (96, 16, 16, 16, 160)   # >= 84 MiB per shard: every shard has the tile path
    boxes, ops = synth.config_queries("C2a", nq=200, extents=ext)
    nq = len(ops)
    dr = torch.from_numpy(boxes.reshape(-1)).cuda()
    do = torch.from_numpy(ops).cuda()
    acc_s = torch.zeros(nq, dtype=torch.int64, device="cuda")
    acc_e = torch.full((2 * nq,), -2 ** 31, dtype=torch.int32, device="cuda")
    used = []
    for g in range(G):
        c = olap.Cube(ext, np.int32, shard=(G, g, b))
        c.fill(olap.GEN_UNIFORM, 23)
        s = torch.empty(nq, dtype=torch.int64, device="cuda")
        e = torch.empty(2 * nq, dtype=torch.int32, device="cuda")
        c.partials_device(dr, do, s, e)
        torch.cuda.synchronize()
        used.append(c.tile_stats()[3])
        olap.combine_partials_device(np.int32, nq, s, e, acc_s, acc_e)
    res = torch.empty(nq * olap.RESULT_DTYPE.itemsize, dtype=torch.uint8, device="cuda")
    olap.finalize_device(ext, np.int32, nq, dr, do, acc_s, acc_e, res)
    torch.cuda.synchronize()
    got = res.cpu().numpy().view(olap.RESULT_DTYPE)
    assert any(used)
    ref = oracle.query(ext, boxes, ops, dtype=np.int32, gen=oracle.GEN_UNIFORM, seed=23,
                       nthreads=oracle.max_threads())
    compare(got, ref, ops, np.int32)


def test_tile_path_full_range_int32_bit_exact():
    """Full-range int32 cells on the tile path (column and wide modes): the biased-cell SUM
    (v ^ 2^31, minus nb * 2^31; reading R7) and MIN/MAX extremes, bit-exact vs the oracle."""
    ext = (40, 16, 16, 16, 160)
    n = int(np.prod(ext))
    rng = np.random.default_rng(31)
    cells = rng.integers(-(2 ** 31), 2 ** 31, size=n, dtype=np.int64).astype(np.int32)
    cells[:2] = [-(2 ** 31), 2 ** 31 - 1]
    c = olap.Cube(ext, np.int32)
    c.load(cells)
    boxes, _ = synth.config_queries("C2a", nq=512, extents=ext, seed=7)
    boxes[0] = [[0, e - 1] for e in ext]
    ops = synth.ops_uniform(len(boxes), rng)
    got = c.query(boxes, ops)
    assert c.tile_stats()[3], "batch expected to take the tile path"
    ref = oracle.query(ext, boxes, ops, cells, nthreads=oracle.max_threads())
    compare(got, ref, ops, np.int32)


def test_tile_workspace_failure_falls_back_to_items(monkeypatch):
    """when the tile workspace cannot grow after a batch took the tile path, the cube
    switches the tile path off and must clear the device's mode word, or every later batch would
    skip the item path and finalize stale partials.  OLAP_TEST_TILE_WS_LIMIT makes the library's
    allocation 'fail' above a query capacity."""
    ext = (32, 16, 16, 16, 192)  # 96 MiB
    seed = 0x5EED2200
    c = olap.Cube(ext, np.float32)
    c.fill(olap.GEN_UNIFORM, seed)
    rng = np.random.default_rng(seed)
    b1 = synth.fraction_boxes(ext, 512, rng, 1e-2, 0.5)
    o1 = synth.ops_mix(512, rng)
    c.query(b1, o1)
    assert c.tile_stats()[3], "first batch should take the tile path"
    monkeypatch.setenv("OLAP_TEST_TILE_WS_LIMIT", "1500")
    b2 = synth.fraction_boxes(ext, 2000, rng, 1e-2, 0.5)
    o2 = synth.ops_mix(2000, rng)
    got = c.query(b2, o2)
    en, _, _, used = c.tile_stats()
    assert not en and not used
    idx = rng.choice(2000, 120, replace=False)
    ref = oracle.query(ext, b2[idx], o2[idx], dtype=np.float32, gen=oracle.GEN_UNIFORM, seed=seed,
                       nthreads=oracle.max_threads())
    compare(got[idx], ref, o2[idx], np.float32)


@pytest.mark.parametrize("ext", [(40, 16, 20, 16, 160), (16, 16, 16, 16, 16, 64), (6, 1400, 2048)])
def test_tile_path_signed_noninteger_float(ext):
    """the tile path's float SUM (slot trees: fp32 trees of <= 256 cells, then
    fp64; reading R8') on mixed-sign, non-integer cells spanning 6 orders of magnitude: within
    1e-6 * sum|x| of the fp64 oracle; MIN / MAX / COUNT exact.  Covers the tree path (runs of > 4
    slots), column mode (<= 4 slots) and edge cells."""
    from test_gpu_parity import compare_signed, signed_cells
    n = int(np.prod(ext))
    cells = signed_cells(n, 0x5EED2300 + n % 997)
    c = olap.Cube(ext, np.float32)
    c.load(cells)
    rng = np.random.default_rng(n % 991)
    boxes = np.concatenate([synth.fraction_boxes(ext, 200, rng, 1e-3, 0.5), synth.random_boxes(ext, 60, rng)])
    ops = synth.ops_uniform(len(boxes), rng)
    got = c.query(boxes, ops)
    assert c.tile_stats()[3], "batch expected to take the tile path"
    compare_signed(got, cells, ext, boxes, ops)
