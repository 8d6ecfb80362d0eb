"""GPU parity: the CUDA path (through the C-ABI) vs the oracle, element by element.

Bars (BASELINE.json north_star):
  * int32 cubes: every field bit-exact (SUM int64 wraparound, COUNT, MIN, MAX, AVG as
    (double)SUM/(double)V computed identically);
  * float32 cubes: COUNT/MIN/MAX exact; SUM/AVG within 1e-6 relative of the fp64
    oracle (north_star), and bit-exact on integer-valued (affine) cubes where every
    fp64 partial sum is exact in any order.
"""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_ipps_malikrse12_b200 as olap
import synth

pytestmark = pytest.mark.gpu

REL = 1e-6   # north_star float tolerance


def compare(gpu, ref, ops, dtype, exact_float=False, rel=REL):
    assert gpu.shape == ref.shape
    assert np.array_equal(gpu["flags"], ref["flags"]), np.nonzero(gpu["flags"] != ref["flags"])[0][:10]
    if dtype == np.int32 or exact_float:
        bad = np.nonzero((gpu["i"] != ref["i"]) | (gpu["d"] != ref["d"]))[0]
        assert bad.size == 0, f"{bad.size} mismatches, first {bad[:5]}: gpu {gpu[bad[:3]]} ref {ref[bad[:3]]}"
        return
    assert np.array_equal(gpu["i"], ref["i"])
    exact = (ops == oracle.MIN) | (ops == oracle.MAX) | (ops == oracle.COUNT)
    assert np.array_equal(gpu["d"][exact], ref["d"][exact])
    tol = rel * np.abs(ref["d"]) + 1e-300
    bad = np.nonzero(np.abs(gpu["d"] - ref["d"]) > tol)[0]
    assert bad.size == 0, f"{bad.size} beyond {rel}: {gpu['d'][bad[:5]]} vs {ref['d'][bad[:5]]}"


def compare_signed(gpu, cells, ext, boxes, ops, bound=1e-6):
    """Mixed-sign, non-integer float32 cells (SURVEY S8 / reading R8'): COUNT, MIN, MAX and the
    flags exact; SUM and AVG within bound * sum|x| of the fp64 oracle (sum|x| = the oracle's SUM
    over |cells|, divided by V for AVG)."""
    ref = oracle.query(ext, boxes, ops, cells, nthreads=oracle.max_threads())
    sums = (ops == oracle.SUM) | (ops == oracle.AVG)
    so = np.where(sums, oracle.SUM, ops).astype(np.int32)
    absref = oracle.query(ext, boxes, so, np.abs(cells), nthreads=oracle.max_threads())
    assert np.array_equal(gpu["flags"], ref["flags"])
    assert np.array_equal(gpu["i"], ref["i"])
    assert np.array_equal(gpu["d"][~sums], ref["d"][~sums])
    V = np.prod(boxes[:, :, 1] - boxes[:, :, 0] + 1, axis=1).astype(np.float64)
    tol = bound * np.where(ops == oracle.AVG, absref["d"] / np.maximum(V, 1), absref["d"]) + 1e-300
    err = np.abs(gpu["d"] - ref["d"])
    bad = np.nonzero(sums & (err > tol))[0]
    assert bad.size == 0, f"{bad.size} beyond {bound}*sum|x|: err {err[bad[:4]]} tol {tol[bad[:4]]}"
    return float(np.max(np.where(sums, err / tol * bound, 0.0)))


def signed_cells(n, seed):
    """float32 cells of both signs over six orders of magnitude, non-integer (no exact sums)."""
    rng = np.random.default_rng(seed)
    return (rng.standard_normal(n) * 10.0 ** rng.uniform(-3, 3, size=n)).astype(np.float32)


def test_hand_example_fig2():
    cells = np.arange(64, dtype=np.int32)
    c = olap.Cube((4, 4, 4), np.int32)
    c.load(cells)
    box = np.array([[[1, 2], [1, 3], [0, 1]]] * 5)
    ops = np.array([olap.COUNT, olap.SUM, olap.MIN, olap.MAX, olap.AVG], np.int32)
    r = c.query(box, ops)
    assert list(r["i"][:4]) == [12, 390, 20, 45] and r["d"][4] == 32.5


def test_c1_full_bit_exact():
    """Config C1: 4-D int32 32^4, 1,000 random boxes, 1 GPU vs the CPU oracle — all bit-exact."""
    cfg = synth.CONFIGS["C1"]
    cells = synth.uniform_cells(int(np.prod(cfg["extents"])), np.int32, cfg["seed"])
    boxes, ops = synth.config_queries("C1")
    c = olap.Cube(cfg["extents"], np.int32)
    c.load(cells)
    gpu = c.query(boxes, ops)
    ref = oracle.query(cfg["extents"], boxes, ops, cells)
    compare(gpu, ref, ops, np.int32)
    # every op on every box
    for op in range(5):
        o = np.full(len(boxes), op, np.int32)
        compare(c.query(boxes, o), oracle.query(cfg["extents"], boxes, o, cells), o, np.int32)



@pytest.mark.parametrize("nq", [1, 4095, 4096, 4097, 16384, 16385])
def test_planner_batch_size_boundaries(nq):
    """Batch sizes around the planner switch: <= 16,384 queries plan in one
    block (plan_small_kernel), larger ones through items_kernel + CUB scan + scan_fix_kernel;
    int32 bit-exact, including empty boxes (lo > hi)."""
    ext = (12, 16, 33)
    cells = synth.uniform_cells(int(np.prod(ext)), np.int32, 1234 + nq)
    rng = np.random.default_rng(nq)
    boxes = synth.random_boxes(ext, nq, rng)
    ops = synth.ops_uniform(nq, rng)
    if nq > 2:
        boxes[nq // 2, 1] = [9, 3]    # lo > hi: empty, reported in flags
        boxes[nq - 1, 2] = [20, 19]
    c = olap.Cube(ext, np.int32)
    c.load(cells)
    compare(c.query(boxes, ops), oracle.query(ext, boxes, ops, cells), ops, np.int32)

SHAPES = [
    ((8, 8, 8, 8, 8, 64), "C2a-like, runs >= 128 cells merge"),
    ((8, 8, 16, 16, 16, 16), "C2b-like, short runs"),
    ((3, 1000), "long rows, vector path with ragged heads/tails"),
    ((5000,), "1-D"),
    ((2, 3, 2, 3, 2, 3, 2, 3), "8-D"),
    ((1, 1, 37), "extent-1 dims"),
    ((64, 129, 7), "odd inner extents"),
    ((17, 4099), "piece boundaries (2048-cell pieces) + tail"),
    ((5, 3, 40), "inner 40: 32-B slots, short runs"),
    ((9, 36), "inner 36: pitch padded to 40 (32-B slots)"),
    ((7, 12), "inner 12: 16-B slots"),
    ((6, 4096), "runs of 512/513 slots: short/long switch"),
    ((3, 5, 8), "runs of 1-2 slots: edge pass only"),
    ((2, 9, 16384), "long runs over several 2048-slot tasks"),
]


@pytest.mark.parametrize("dtype", [np.int32, np.float32])
@pytest.mark.parametrize("ext,why", SHAPES)
def test_shapes_random_and_fraction_boxes(ext, why, dtype):
    n = int(np.prod(ext))
    seed = 0x5EED1000 + n
    cells = synth.uniform_cells(n, dtype, seed)
    rng = np.random.default_rng(seed)
    b1 = synth.random_boxes(ext, 300, rng)
    b2 = synth.fraction_boxes(ext, 300, rng, 1e-4)
    full = np.array([[[0, e - 1] for e in ext]])
    boxes = np.concatenate([b1, b2, full, full])
    ops = synth.ops_uniform(len(boxes), rng)
    ops[-2:] = [olap.SUM, olap.MIN]
    c = olap.Cube(ext, dtype)
    c.load(cells)
    compare(c.query(boxes, ops), oracle.query(ext, boxes, ops, cells), ops, dtype)


@pytest.mark.parametrize("dtype", [np.int32, np.float32])
def test_affine_integer_valued_bit_exact(dtype):
    """Integer-valued affine cube: fp64 sums are exact in any order -> float32 SUM/AVG bit-exact too."""
    ext = (12, 10, 9, 300)
    params = np.array([7, 3, -2, 5, 1], float)
    c = olap.Cube(ext, dtype)
    c.fill(olap.GEN_AFFINE, 0, params)
    rng = np.random.default_rng(5)
    boxes = np.concatenate([synth.random_boxes(ext, 400, rng), synth.fraction_boxes(ext, 400, rng, 1e-4)])
    ops = synth.ops_uniform(len(boxes), rng)
    ref = oracle.query(ext, boxes, ops, dtype=dtype, gen=oracle.GEN_AFFINE, params=params)
    compare(c.query(boxes, ops), ref, ops, dtype, exact_float=True)


def test_fill_matches_inputs_generator():
    """The device generator equals the seeded input generator (same published splitmix64
    formula), read back cell by cell through 1-cell MAX queries."""
    for dtype in (np.int32, np.float32):
        ext = (33, 70)
        c = olap.Cube(ext, dtype)
        c.fill(olap.GEN_UNIFORM, 0x5EED0001)
        xs, ys = np.meshgrid(np.arange(33), np.arange(70), indexing="ij")
        boxes = np.stack([np.stack([xs.ravel(), xs.ravel()], -1), np.stack([ys.ravel(), ys.ravel()], -1)], 1)
        r = c.query(boxes, np.full(len(boxes), olap.MAX, np.int32))
        got = r["i"].astype(np.int32) if dtype == np.int32 else r["d"].astype(np.float32)
        assert np.array_equal(got, synth.uniform_cells(33 * 70, dtype, 0x5EED0001))


def test_c2_full_size_sampled():
    """Config C2a at full size (1 GiB float32, 4,096-query batch, the bench's launch
    configuration): GPU vs oracle on a sample of queries the oracle recomputes one by one."""
    cfg = synth.CONFIGS["C2a"]
    ext = cfg["extents"]
    c = olap.Cube(ext, np.float32)
    c.fill(olap.GEN_UNIFORM, cfg["seed"])
    boxes, ops = synth.config_queries("C2a")
    gpu = c.query(boxes, ops)
    rng = np.random.default_rng(0)
    # sample: smallest, largest and random queries (bounded oracle work)
    vol = np.prod(boxes[:, :, 1] - boxes[:, :, 0] + 1, axis=1)
    idx = np.unique(np.concatenate([np.argsort(vol)[:12], rng.choice(len(boxes), 24, replace=False)]))
    idx = idx[vol[idx] < 60_000_000][:30]
    ref = oracle.query(ext, boxes[idx], ops[idx], dtype=np.float32, gen=oracle.GEN_UNIFORM, seed=cfg["seed"],
                       nthreads=oracle.max_threads())
    compare(gpu[idx], ref, ops[idx], np.float32)
    # the full-cube answer of an integer-valued affine fill is exact
    params = np.array([1, 3, 5, 7, 11, 13, 1], float)
    c.fill(olap.GEN_AFFINE, 0, params)
    full = np.array([[[0, e - 1] for e in ext]] * 3)
    o3 = np.array([olap.SUM, olap.MIN, olap.MAX], np.int32)
    V = int(np.prod(ext))
    s = V * 1 + sum(int(params[1 + d]) * (V // ext[d]) * ((ext[d] - 1) * ext[d] // 2) for d in range(6))
    g3 = c.query(full, o3)
    assert g3["d"][0] == float(s) and g3["d"][1] == 1.0
    assert g3["d"][2] == 1 + sum(int(params[1 + d]) * (ext[d] - 1) for d in range(6))
    # and on a sample of the batch against the oracle, bit-exact
    gpu = c.query(boxes, ops)
    idx2 = idx[:12]
    ref2 = oracle.query(ext, boxes[idx2], ops[idx2], dtype=np.float32, gen=oracle.GEN_AFFINE, params=params,
                        nthreads=oracle.max_threads())
    compare(gpu[idx2], ref2, ops[idx2], np.float32, exact_float=True)


def test_c2_full_size_top_decile():
    """the largest boxes of the full-size C2a batch (the top decile by volume
    holds ~3/4 of the batch's algorithmic bytes) against the OpenMP oracle on the random fill, and
    bit-exact on the integer-valued affine fill -- the boxes the sampled test above leaves out."""
    cfg = synth.CONFIGS["C2a"]
    ext = cfg["extents"]
    c = olap.Cube(ext, np.float32)
    c.fill(olap.GEN_UNIFORM, cfg["seed"])
    boxes, ops = synth.config_queries("C2a")
    gpu = c.query(boxes, ops)
    assert c.tile_stats()[3]
    vol = np.prod(boxes[:, :, 1] - boxes[:, :, 0] + 1, axis=1)
    top = np.argsort(vol)[::-1][:len(vol) // 10]
    rng = np.random.default_rng(1)
    idx = np.unique(np.concatenate([top[:24], rng.choice(top, 24, replace=False)]))
    ref = oracle.query(ext, boxes[idx], ops[idx], dtype=np.float32, gen=oracle.GEN_UNIFORM, seed=cfg["seed"],
                       nthreads=oracle.max_threads())
    compare(gpu[idx], ref, ops[idx], np.float32)
    params = np.array([1, 3, 5, 7, 11, 13, 1], float)
    c.fill(olap.GEN_AFFINE, 0, params)
    gpu = c.query(boxes, ops)
    ref2 = oracle.query(ext, boxes[idx], ops[idx], dtype=np.float32, gen=oracle.GEN_AFFINE, params=params,
                        nthreads=oracle.max_threads())
    compare(gpu[idx], ref2, ops[idx], np.float32, exact_float=True)


@pytest.mark.parametrize("ext", [(16, 16, 16, 16, 16, 16), (16, 16, 16, 16, 16, 48)])
def test_determinism_float_sums(ext):
    """Float sums are bit-stable run to run, with and without the L2-aware item order
    (the 192 MiB cube takes it): blocks pick items up in a different order every run,
    but partials are folded in item order."""
    c = olap.Cube(ext, np.float32)
    c.fill(olap.GEN_UNIFORM, 99)
    assert c.stats()[1] == (int(np.prod(ext)) * 4 > (64 << 20))
    boxes, ops = synth.config_queries("C2a", nq=2048, extents=ext)
    a = c.query(boxes, ops)
    for _ in range(3):
        assert c.query(boxes, ops).tobytes() == a.tobytes()


def test_empty_invalid_and_errors():
    ext = (6, 7, 8)
    cells = synth.uniform_cells(6 * 7 * 8, np.int32, 3)
    c = olap.Cube(ext, np.int32)
    c.load(cells)
    boxes = np.array([[[2, 1], [0, 6], [0, 7]], [[0, 5], [3, 3], [8, 7]], [[0, 0], [0, 0], [0, 0]]])
    ops = np.array([olap.SUM, olap.MAX, olap.MIN], np.int32)
    r = c.query(boxes, ops)
    assert list(r["flags"]) == [olap.RESULT_EMPTY, olap.RESULT_EMPTY, 0]
    assert r["i"][2] == cells[0]
    with pytest.raises(olap.OlapError) as ei:
        c.query(np.array([[[0, 6], [0, 6], [0, 7]]]), [olap.SUM])
    assert ei.value.status == olap.E_RANGE and "query 0 dimension 0" in str(ei.value)
    with pytest.raises(olap.OlapError):
        c.query(np.array([[[0, 1], [0, 1], [0, 1]]]), [9])
    assert c.query(np.zeros((0, 3, 2), np.int64), np.zeros(0, np.int32)).shape == (0,)
    # device path flags invalid queries instead of failing the batch
    dr = torch.tensor(np.array([[[0, 6], [0, 6], [0, 7]], [[0, 5], [0, 6], [0, 7]], [[0, 1], [0, 1], [0, 1]]]),
                      dtype=torch.int64, device="cuda")
    do = torch.tensor([olap.SUM, olap.SUM, 7], dtype=torch.int32, device="cuda")
    res = torch.empty(3 * 24, dtype=torch.uint8, device="cuda")
    c.query_device(dr, do, res)
    out = res.cpu().numpy().view(olap.RESULT_DTYPE)
    assert list(out["flags"]) == [olap.RESULT_INVALID, 0, olap.RESULT_INVALID]
    assert out["i"][1] == int(cells.astype(np.int64).sum())


@pytest.mark.parametrize("G,b", [(2, 1), (3, 2), (4, 1), (8, 16), (5, 3)])
@pytest.mark.parametrize("dtype", [np.int32, np.float32])
def test_virtual_shards_combine_to_global(G, b, dtype):
    """G shards of one cube on one GPU: shard partials + the exchange's reduction
    (olap_partials_combine_device) + finalize == the unsharded answer / the oracle."""
    ext = (64, 9, 130)
    n = int(np.prod(ext))
    cells = synth.uniform_cells(n, dtype, 0x5EED2000 + G)
    rng = np.random.default_rng(G * 10 + b)
    boxes = np.concatenate([synth.random_boxes(ext, 400, rng), synth.fraction_boxes(ext, 200, rng, 1e-3)])
    ops = synth.ops_uniform(len(boxes), rng)
    nq = len(boxes)
    dr = torch.from_numpy(boxes.astype(np.int64)).cuda()
    do = torch.from_numpy(ops).cuda()
    acc_s = torch.zeros(nq, dtype=torch.int64, device="cuda")
    acc_e = torch.full((2 * nq,), -(2 ** 31), dtype=torch.int32, device="cuda")
    shards = []
    for g in range(G):
        cg = olap.Cube(ext, dtype, shard=(G, g, b))
        cg.load(cells)
        shards.append(cg)
        s = torch.empty(nq, dtype=torch.int64, device="cuda")
        e = torch.empty(2 * nq, dtype=torch.int32, device="cuda")
        cg.partials_device(dr, do, s, e)
        olap.combine_partials_device(dtype, nq, s, e, acc_s, acc_e)
    res = torch.empty(nq * 24, dtype=torch.uint8, device="cuda")
    olap.finalize_device(ext, dtype, nq, dr, do, acc_s, acc_e, res)
    got = res.cpu().numpy().view(olap.RESULT_DTYPE)
    ref = oracle.query(ext, boxes, ops, cells)
    compare(got, ref, ops, dtype, rel=1e-12)
    # a shard filled on the device holds the right global cells
    cg = olap.Cube(ext, dtype, shard=(G, G - 1, b))
    cg.fill(olap.GEN_UNIFORM, 0x5EED2000 + G)
    s = torch.empty(nq, dtype=torch.int64, device="cuda")
    e = torch.empty(2 * nq, dtype=torch.int32, device="cuda")
    cg.partials_device(dr, do, s, e)
    s2 = torch.empty_like(s)
    e2 = torch.empty_like(e)
    shards[G - 1].partials_device(dr, do, s2, e2)
    assert torch.equal(s, s2) and torch.equal(e, e2)


# ------------------------------------------------------------------ dictionaries

def test_dict_translate_parity():
    keys = synth.random_keys(20000, seed=1, min_len=0, max_len=40)
    d = olap.Dict(keys)
    od = oracle.Dict(keys)
    assert len(d) == len(od)
    probes = keys[::3] + synth.random_keys(5000, seed=2, min_len=0, max_len=40) + [k + b"\0" for k in keys[:200]]
    ids, miss = d.translate(probes)
    ref = od.translate(probes)
    assert np.array_equal(ids, ref)
    assert miss == int((ref < 0).sum())
    for i in [0, 1, len(d) // 2, len(d) - 1]:
        assert d.lookup(i) == od.lookup(i)


def test_dict_multi_and_bounds():
    members = synth.tpcds_members()
    cols = list(members)
    dg = [olap.Dict(members[c]) for c in cols]
    do = [oracle.Dict(members[c]) for c in cols]
    rng = np.random.default_rng(4)
    which = rng.integers(0, 4, size=3000).astype(np.int32)
    keys = []
    for w in which:
        m = members[cols[w]]
        k = m[rng.integers(0, len(m))]
        keys.append(k if rng.random() < 0.9 else k[:-1])
    ids, miss = olap.translate(dg, which, keys)
    ref = np.array([do[w].translate([k])[0] for w, k in zip(which, keys)], np.int32)
    assert np.array_equal(ids, ref) and miss == int((ref < 0).sum())
    probes = ["1997-01-01", "1998-01-01", "1999-02-29", "2000-02-29", "2002-12-31", "2003", "", "2001-06-15x"]
    for upper in (False, True):
        got = dg[0].bound(probes, upper=upper)
        assert list(got) == [do[0].bound(p, upper=upper) for p in probes]


def test_dict_stress_1e6():
    keys = synth.random_keys(1_000_000, seed=7, min_len=4, max_len=20, alphabet=b"abcdefghij")
    d = olap.Dict(keys)
    od = oracle.Dict(keys)
    probes = keys[::5] + synth.random_keys(100_000, seed=8, min_len=4, max_len=20, alphabet=b"abcdefghij")
    ids, _ = d.translate(probes)
    assert np.array_equal(ids, od.translate(probes))


def _expected_range(od, cond, n):
    """Reading R11/R13 applied to the oracle dictionary's answers."""
    if cond is None:
        return (0, n - 1), 0
    if isinstance(cond, tuple):
        return (od.bound(cond[0]), od.bound(cond[1], upper=True) - 1), 0
    i = int(od.translate([cond])[0])
    return ((i, i), 0) if i >= 0 else ((1, 0), 1)


def test_text_ranges_parity():
    members = synth.tpcds_members()
    cols = ["ca_state", "i_class", "s_store_id", "d_date"]
    dg = [olap.Dict(members[c]) for c in cols]
    do = [oracle.Dict(members[c]) for c in cols]
    ext = [len(members[c]) for c in cols]
    rng = np.random.default_rng(9)
    conds = []
    for _ in range(3000):
        q = []
        for di, c in enumerate(cols):
            m = members[c]
            r = rng.random()
            if r < 0.3:
                q.append(None)
            elif r < 0.65:
                k = m[rng.integers(0, len(m))]
                q.append(k if rng.random() < 0.9 else k + "~")
            else:
                a, b = sorted(rng.integers(0, len(m), size=2))
                s1, s2 = m[a], m[b]
                if rng.random() < 0.3:
                    s1 = s1[:-1]          # endpoint not a member
                if rng.random() < 0.3:
                    s2 = s2 + "zz"
                if rng.random() < 0.05:
                    s1, s2 = s2, s1       # reversed -> empty
                q.append((s1, s2))
        conds.append(q)
    got, miss = olap.text_ranges(dg, ext, conds)
    want = np.zeros_like(got)
    wmiss = 0
    for qi, q in enumerate(conds):
        for di in range(4):
            (lo, hi), m = _expected_range(do[di], q[di], ext[di])
            want[qi, di] = (lo, hi)
            wmiss += m
    assert np.array_equal(got, want)
    assert miss == wmiss
    # mixed numeric (IDS) dimension and a dimension without a dictionary
    got2, _ = olap.text_ranges([dg[0], None], [ext[0], 10], [["CA", ("ids", 2, 5)], [None, None]])
    assert got2.tolist() == [[[int(do[0].translate(["CA"])[0])] * 2, [2, 5]], [[0, ext[0] - 1], [0, 9]]]
    with pytest.raises(olap.OlapError):
        olap.text_ranges([dg[0], None], [ext[0], 10], [["CA", "x"]])   # text on a dim without dictionary


@pytest.mark.parametrize("dtype", [np.int32, np.float32])
@pytest.mark.parametrize("shard", [None, (3, 1, 2)])
def test_add_facts_builds_cube(dtype, shard):
    ext = (13, 7, 11)
    rng = np.random.default_rng(2)
    nrows = 50_000
    ids = np.stack([rng.integers(0, n, size=nrows) for n in ext]).astype(np.int32)
    vals = rng.integers(-1000, 1000, size=nrows).astype(dtype)
    ref = np.zeros(ext, np.int64)
    np.add.at(ref, tuple(ids), vals.astype(np.int64))
    refn = np.zeros(ext, np.int64)
    np.add.at(refn, tuple(ids), 1)
    G = 1 if shard is None else shard[0]
    for cube_ref, v in ((ref, vals), (refn, None)):
        c = olap.Cube(ext, dtype, shard=shard)
        c.fill(olap.GEN_AFFINE, 0, np.zeros(4))
        c.add_facts_device(torch.from_numpy(ids).cuda(), None if v is None else torch.from_numpy(v).cuda())
        torch.cuda.synchronize()
        # every cell through 1-cell SUM queries (partials of this shard; non-owned rows are identity)
        boxes = np.array([[[x, x], [y, y], [z, z]] for x in range(ext[0]) for y in range(ext[1])
                          for z in range(ext[2])])
        nq = len(boxes)
        s = torch.empty(nq, dtype=torch.int64, device="cuda")
        e = torch.empty(2 * nq, dtype=torch.int32, device="cuda")
        c.partials_device(torch.from_numpy(boxes).cuda(), torch.full((nq,), olap.SUM, dtype=torch.int32,
                                                                   device="cuda"), s, e)
        got = s.cpu().numpy()
        if dtype == np.float32:
            got = got.view(np.float64)
        owned = np.array([((x // shard[2]) % G == shard[1]) if shard else True for x, _, _ in
                          (b[:, 0] for b in boxes)])
        want = cube_ref.reshape(-1).astype(np.float64 if dtype == np.float32 else np.int64)
        assert np.array_equal(got[owned], want[owned])
        assert not got[~owned].any()


def test_c4_tpcds_pipeline():
    """C4 end to end: fact rows -> GPU cube build (quantity, count) -> string predicates ->
    GPU translation into ranges (4 dictionaries) -> cube queries, equal to the oracle's fact
    scan over the raw rows (SUM of quantity, fact COUNT)."""
    members = synth.tpcds_members()
    cols = ["ca_state", "i_class", "s_store_id", "d_date"]   # layout: date innermost
    nrows = 400_000
    facts, qty, cents = synth.tpcds_facts(nrows, members)
    dg = [olap.Dict(members[c]) for c in cols]
    do = {c: oracle.Dict(members[c]) for c in cols}
    # fact rows -> ids (GPU translation of the raw strings, checked against the oracle on a sample)
    ids = []
    for di, c in enumerate(cols):
        strs = [members[c][i] for i in facts[c][:20000]]
        g, _ = dg[di].translate(strs)
        assert np.array_equal(g, do[c].translate(strs))
        ids.append(do[c].translate([members[c][i] for i in range(len(members[c]))])[facts[c]])
    ids = np.stack(ids).astype(np.int32)
    ext = tuple(len(members[c]) for c in cols)
    d_ids = torch.from_numpy(ids).cuda()
    cq = olap.Cube(ext, np.int32)
    cq.fill(olap.GEN_AFFINE, 0, np.zeros(5))
    cq.add_facts_device(d_ids, torch.from_numpy(qty).cuda())
    cn = olap.Cube(ext, np.int32)
    cn.fill(olap.GEN_AFFINE, 0, np.zeros(5))
    cn.add_facts_device(d_ids)
    torch.cuda.synchronize()
    queries = synth.tpcds_queries(300, members)
    conds = [[q.get(c) if c != "d_date" else q[c] for c in cols] for q in queries]
    boxes, _ = olap.text_ranges(dg, ext, conds)
    sums = cq.query(boxes, np.full(len(boxes), olap.SUM, np.int32))
    cnts = cn.query(boxes, np.full(len(boxes), olap.SUM, np.int32))
    # the oracle path: its own dictionaries on the raw strings, then a scan over the fact rows
    ob = np.zeros_like(boxes)
    for qi, cond in enumerate(conds):
        for di, c in enumerate(cols):
            ob[qi, di] = _expected_range(do[c], cond[di], ext[di])[0]
    ref_s, ref_c = oracle.factscan(ids, qty, ob)
    assert np.array_equal(sums["i"], ref_s)
    assert np.array_equal(cnts["i"], ref_c)


def _sampled_full_size(name, n_small, n_random, max_cells, affine_params, layout=olap.LAYOUT_ROWMAJOR):
    cfg = synth.CONFIGS[name]
    ext = cfg["extents"]
    c = olap.Cube(ext, cfg["dtype"], layout=layout)
    try:
        c.fill(olap.GEN_UNIFORM, cfg["seed"])
        boxes, ops = synth.config_queries(name)
        gpu = c.query(boxes, ops)
        vol = np.prod(boxes[:, :, 1] - boxes[:, :, 0] + 1, axis=1)
        rng = np.random.default_rng(1)
        cand = np.nonzero(vol <= max_cells)[0]
        idx = np.unique(np.concatenate([np.argsort(vol)[:n_small], rng.choice(cand, min(n_random, len(cand)),
                                                                                replace=False)]))
        ref = oracle.query(ext, boxes[idx], ops[idx], dtype=cfg["dtype"], gen=oracle.GEN_UNIFORM, seed=cfg["seed"],
                           nthreads=oracle.max_threads())
        compare(gpu[idx], ref, ops[idx], cfg["dtype"])
        # integer-valued affine fill: float results bit-exact on a sample incl. large boxes
        c.fill(olap.GEN_AFFINE, 0, affine_params)
        gpu = c.query(boxes, ops)
        ref = oracle.query(ext, boxes[idx], ops[idx], dtype=cfg["dtype"], gen=oracle.GEN_AFFINE,
                           params=affine_params, nthreads=oracle.max_threads())
        compare(gpu[idx], ref, ops[idx], cfg["dtype"], exact_float=True)
    finally:
        c.close()


def test_c3_full_size_sampled():
    """C3: 32 GiB float32 cube (2048^3), 4,096-query batch; sampled oracle parity."""
    _sampled_full_size("C3", 12, 12, 150_000_000, np.array([1, 1, 2, 3], float))


def test_c5_slice_full_size_sampled():
    """C5 per-GPU slice: 128 GiB float32 cube (1024,4096,8192), 65,536 small boxes; sampled parity."""
    _sampled_full_size("C5", 50, 400, 2_000_000, np.array([2, 1, 1, 1], float))


def test_c5_slice_bricked_full_size_sampled():
    """C5 as bench.py runs it: the 128 GiB slice in the bricked layout (R26)."""
    _sampled_full_size("C5", 50, 400, 2_000_000, np.array([2, 1, 1, 1], float), layout=olap.LAYOUT_BRICK3)


# ------------------------------------------------------------------ fact tables (NEXT #1)

def _table_cols(nrows, rng):
    dims = [rng.integers(0, n, size=nrows).astype(np.int32) for n in (40, 7, 13, 5)]
    qty = rng.integers(-50, 100, size=nrows).astype(np.int32)
    paid = rng.random(nrows).astype(np.float32)
    return dims + [qty, paid]


def _table_queries(rng, nq):
    qs = []
    for _ in range(nq):
        conds = []
        for c, n in enumerate((40, 7, 13, 5)):
            if rng.random() < 0.6:
                a, b = sorted(rng.integers(-2, n + 2, size=2))
                if rng.random() < 0.05:
                    a, b = b + 1, a
                conds.append((c, int(a), int(b)))
        qs.append((conds, int(rng.integers(4, 6)), int(rng.integers(0, 5))))
    return qs


@pytest.mark.parametrize("nrows", [1, 1000, 1024, 5000, 300_001])
def test_table_scan_parity(nrows):
    """Q_D over a column store (Eq. 11-12): GPU shared scan vs oracle.tablescan."""
    rng = np.random.default_rng(nrows)
    cols = _table_cols(nrows, rng)
    t = olap.Table(nrows, [c.dtype for c in cols])
    for i, c in enumerate(cols):
        t.load_column(i, c)
    qs = _table_queries(rng, 500)
    qs.append(([], 4, olap.SUM))                          # no condition: whole column
    qs.append(([(0, 10, 10), (0, 11, 11)], 5, olap.AVG))  # contradictory -> empty
    got = t.query(qs)
    ref = oracle.tablescan(cols, qs, nthreads=oracle.max_threads())
    ops = np.array([q[2] for q in qs], np.int32)
    isf = np.array([cols[q[1]].dtype == np.float32 for q in qs])
    assert np.array_equal(got["flags"], ref["flags"]) and np.array_equal(got["i"], ref["i"])
    ex = ~isf | (ops == olap.MIN) | (ops == olap.MAX) | (ops == olap.COUNT)
    assert np.array_equal(got["d"][ex], ref["d"][ex])
    tol = 1e-6 * np.abs(ref["d"]) + 1e-300
    assert (np.abs(got["d"] - ref["d"]) <= tol).all()
    with pytest.raises(olap.OlapError):
        t.query([([(5, 0, 1)], 4, olap.SUM)])             # condition on a float column


def test_table_scan_chunks_and_long_conditions():
    """The scan keeps 256-query chunks in shared memory with their first 4 conditions inline:
    batches of 1 .. 1,300 queries (ragged last chunk) and queries with 5-9 conditions (the rest
    read from the query descriptor) against oracle.tablescan."""
    nrows = 70_001
    rng = np.random.default_rng(77)
    cols = _table_cols(nrows, rng)
    t = olap.Table(nrows, [c.dtype for c in cols])
    for i, c in enumerate(cols):
        t.load_column(i, c)
    qs = _table_queries(rng, 1300)
    for k in range(0, 1300, 7):  # every 7th query: 5-9 conditions, repeated columns narrowing the range
        conds = []
        for j in range(5 + k % 5):
            c = j % 4
            n = (40, 7, 13, 5)[c]
            conds.append((c, int(rng.integers(-1, 2 + j % 3)), int(n - rng.integers(0, 2 + j % 3))))
        qs[k] = (conds, int(rng.integers(4, 6)), int(rng.integers(0, 5)))
    for nq in (1, 255, 256, 257, 1300):
        sub = qs[:nq]
        got = t.query(sub)
        ref = oracle.tablescan(cols, sub, nthreads=oracle.max_threads())
        ops = np.array([q[2] for q in sub], np.int32)
        isf = np.array([cols[q[1]].dtype == np.float32 for q in sub])
        assert np.array_equal(got["flags"], ref["flags"]) and np.array_equal(got["i"], ref["i"]), nq
        ex = ~isf | (ops == olap.MIN) | (ops == olap.MAX) | (ops == olap.COUNT)
        assert np.array_equal(got["d"][ex], ref["d"][ex]), nq
        assert (np.abs(got["d"] - ref["d"]) <= 1e-6 * np.abs(ref["d"]) + 1e-300).all(), nq
    # deterministic: the same batch twice gives bit-identical results
    assert np.array_equal(t.query(qs).view(np.uint8), t.query(qs).view(np.uint8))


# ------------------------------------------------------------------ multi-resolution cube set (NEXT #3)

def _hier(rng):
    return [synth.date_hierarchy(), synth.random_hierarchy(37, 3, rng), synth.random_hierarchy(50, 3, rng)]


@pytest.mark.parametrize("dtype", [np.int32, np.float32])
def test_rollup_parity(dtype):
    rng = np.random.default_rng(31)
    ids = _hier(rng)
    h = olap.Hierarchy(ids)
    fine_ext = h.extents(2)
    cells = (rng.integers(-1000, 1000, size=fine_ext) if dtype == np.int32 else
             rng.random(fine_ext)).astype(dtype)
    fine = olap.Cube(fine_ext, dtype)
    fine.load(cells)
    for rc in (0, 1):
        for op in (olap.SUM, olap.MIN, olap.MAX):
            ce = h.extents(rc)
            coarse = olap.Cube(ce, dtype)
            h.rollup(fine, 2, coarse, rc, op)
            want = oracle.rollup(ids, cells, 2, rc, op)
            # read every coarse cell back through 1-cell MAX queries
            boxes = np.stack(np.meshgrid(*[np.arange(n) for n in ce], indexing="ij"), -1).reshape(-1, 3)
            boxes = np.repeat(boxes[:, :, None], 2, axis=2)
            r = coarse.query(boxes, np.full(len(boxes), olap.MAX, np.int32))
            got = r["i"].astype(np.int32) if dtype == np.int32 else r["d"].astype(np.float32)
            assert np.array_equal(got, want.ravel()), (rc, op)


def test_cubeset_routing_eq2():
    rng = np.random.default_rng(32)
    ids = _hier(rng)
    h = olap.Hierarchy(ids)
    cells = rng.integers(0, 1000, size=h.extents(2)).astype(np.int32)
    cubes = {2: olap.Cube(h.extents(2), np.int32)}
    cubes[2].load(cells)
    cubes[0] = olap.Cube(h.extents(0), np.int32)
    h.rollup(cubes[2], 2, cubes[0], 0, olap.SUM)
    cs = olap.CubeSet(h)
    cs.add(2, cubes[2])
    cs.add(0, cubes[0])                     # level 1 deliberately missing
    nq = 600
    levels = rng.integers(0, 3, size=(nq, 3)).astype(np.int32)
    ranges = np.zeros((nq, 3, 2), np.int64)
    for q in range(nq):
        for d in range(3):
            n = int(ids[d][levels[q, d]].max()) + 1
            ranges[q, d] = sorted(rng.integers(0, n, size=2))
    ops = synth.ops_uniform(nq, rng)
    got, used = cs.query(ranges, levels, ops)
    R = levels.max(axis=1)
    coarse_cells = oracle.rollup(ids, cells, 2, 0)
    for q in range(nq):
        if R[q] == 1 and ops[q] != olap.SUM:
            assert used[q] == -1 and got["flags"][q] == olap.RESULT_INVALID
            continue
        tgt = R[q] if R[q] != 1 else 2             # SUM at level 1 falls through to the finest cube
        assert used[q] == tgt
        box = np.array([oracle.convert_range(ids[d], int(levels[q, d]), int(tgt), *ranges[q, d]) for d in range(3)])
        src = cells if tgt == 2 else coarse_cells
        ref = oracle.query(src.shape, box[None], ops[q:q + 1], src.ravel())
        assert got[q:q + 1].tobytes() == ref.tobytes(), q
    # SUM is the same at every resolution that can answer it (roll-up preserves sums)
    ext0 = h.extents(0)
    r0 = np.stack([np.sort(rng.integers(0, n, size=(nq, 2)), axis=1) for n in ext0], axis=1)
    sums, used0 = cs.query(r0, np.zeros_like(levels), np.full(nq, olap.SUM, np.int32))
    assert (used0 == 0).all()
    fine_box = h.convert(r0, np.zeros_like(levels), 2)
    direct = cubes[2].query(fine_box, np.full(nq, olap.SUM, np.int32))
    assert np.array_equal(sums["i"], direct["i"])


# ------------------------------------------------------------------ robustness

def test_out_of_memory_is_an_error_not_a_crash():
    # 2^40 float32 cells = 4 TiB: cudaMalloc fails -> OLAP_E_NOMEM, and the device stays usable
    with pytest.raises(olap.OlapError) as ei:
        olap.Cube((1 << 10, 1 << 10, 1 << 20), np.float32)
    assert ei.value.status == olap.E_NOMEM
    c = olap.Cube((4, 4), np.int32)
    c.load(np.arange(16, dtype=np.int32))
    assert c.query(np.array([[[0, 3], [0, 3]]]), [olap.SUM])["i"][0] == 120


def test_concurrent_queries_one_cube():
    """Several host threads query one cube at once: calls serialize on the cube's mutex
    and its workspace event; every thread gets its own correct answers."""
    import threading
    ext = (16, 16, 16, 16, 16, 48)   # > 64 MiB: the L2-ordered path
    c = olap.Cube(ext, np.float32)
    c.fill(olap.GEN_UNIFORM, 5)
    batches = [synth.config_queries("C2a", nq=256, seed=900 + i, extents=ext) for i in range(6)]
    want = [c.query(b, o) for b, o in batches]
    got = [None] * 6

    def run(i):
        for _ in range(3):
            got[i] = c.query(*batches[i])

    th = [threading.Thread(target=run, args=(i,)) for i in range(6)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    for i in range(6):
        assert got[i].tobytes() == want[i].tobytes()


def test_dict_stress_1e7():
    """SURVEY §8(a) a2 stress size: 10^7 keys (16-byte ids), translated on the GPU."""
    rng = np.random.default_rng(77)
    ids = rng.integers(0, 1 << 62, size=10_000_000, dtype=np.int64)
    keys = [b"%016x" % int(v) for v in ids[:2_000_000]]   # 16-char keys; the host build sorts them
    keys += [bytes(8) + int(v).to_bytes(8, "little") for v in ids[2_000_000:]]
    d = olap.Dict(keys)
    assert len(d) == len(set(keys))
    probe_idx = rng.integers(0, len(keys), size=200_000)
    probes = [keys[i] for i in probe_idx] + [b"%016x" % int(v) + b"!" for v in ids[:10_000]]
    got, miss = d.translate(probes)
    assert miss == 10_000
    # ids are ranks in byte order: check against a sorted copy of the distinct keys
    s = sorted(set(keys))
    for k in range(0, 200_000, 997):
        assert s[got[k]] == probes[k]
    assert (got[200_000:] == -1).all()


def test_translate_device_counts_misses_on_device():
    d = olap.Dict(["a", "bb", "ccc"])
    keys = [b"a", b"x", b"ccc", b"bb", b""]
    buf = np.frombuffer(b"".join(keys), np.uint8).copy()
    offs = np.concatenate([[0], np.cumsum([len(k) for k in keys])]).astype(np.int64)
    dbuf = torch.from_numpy(buf).cuda()
    doff = torch.from_numpy(offs).cuda()
    ids = torch.empty(len(keys), dtype=torch.int32, device="cuda")
    miss = torch.zeros(1, dtype=torch.int64, device="cuda")
    olap.translate_device([d], None, dbuf, doff, len(keys), ids, miss)
    torch.cuda.synchronize()
    assert ids.cpu().tolist() == [0, -1, 2, 1, -1] and int(miss.item()) == 2


def test_cuda_graph_capture_replay():
    """olap_query_batch_device captured into a CUDA graph (after a warm-up call sized the
    workspace) replays to the same bytes as direct calls, on the L2-ordered path too."""
    for ext in ((16, 16, 16, 16), (16, 16, 16, 16, 16, 48)):
        c = olap.Cube(ext, np.float32)
        c.fill(olap.GEN_UNIFORM, 3)
        boxes, ops = synth.config_queries("C2a", nq=512, seed=5, extents=ext)
        dr = torch.from_numpy(boxes).cuda()
        do = torch.from_numpy(ops).cuda()
        res = torch.zeros(512 * 24, dtype=torch.uint8, device="cuda")
        st = torch.cuda.Stream()
        with torch.cuda.stream(st):
            c.query_device(dr, do, res, stream=st)           # warm-up sizes the workspace
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
        big = torch.from_numpy(np.concatenate([boxes] * 8)).cuda()   # 4,096 > the 1,024-query workspace
        with pytest.raises(olap.OlapError):                            # cannot grow inside a capture
            g2 = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g2, stream=st):
                c.query_device(big, torch.cat([do] * 8), torch.zeros(4096 * 24, dtype=torch.uint8, device="cuda"),
                               stream=torch.cuda.current_stream())


@pytest.mark.parametrize("ext", [(9, 40, 33), (5, 7, 1000), (3, 3, 3, 64)])
def test_full_range_int32_cells(ext):
    """int32 cells over the whole int32 range: SUM of biased cells (v ^ 2^31) minus nb * 2^31
    (int64 mod 2^64, R7), MIN/MAX at the extremes, AVG = SUM/V — bit-exact vs the oracle, on
    the row-major item / tile paths and the bricked layout."""
    rng = np.random.default_rng(int(np.prod(ext)))
    n = int(np.prod(ext))
    cells = rng.integers(-(2 ** 31), 2 ** 31, size=n, dtype=np.int64).astype(np.int32)
    cells[:3] = [-(2 ** 31), 2 ** 31 - 1, 0]
    boxes = np.concatenate([synth.random_boxes(ext, 300, rng), np.array([[[0, e - 1] for e in ext]])])
    for layout in (olap.LAYOUT_ROWMAJOR, olap.LAYOUT_BRICK):
        c = olap.Cube(ext, np.int32, layout=layout)
        c.load(cells)
        for op in range(5):
            ops = np.full(len(boxes), op, np.int32)
            compare(c.query(boxes, ops), oracle.query(ext, boxes, ops, cells), ops, np.int32)
        c.close()


def test_text_ranges_device_matches_host():
    members = synth.tpcds_members()
    cols = ["ca_state", "i_class", "s_store_id", "d_date"]
    dg = [olap.Dict(members[c]) for c in cols]
    ext = [len(members[c]) for c in cols]
    qs = synth.tpcds_queries(2000, members, seed=123)
    conds = [[q.get(c) if c != "d_date" else q[c] for c in cols] for q in qs]
    want, wmiss = olap.text_ranges(dg, ext, conds)
    kinds, first, rin, buf, offs = olap.pack_text_conditions(conds, 4)
    out = torch.empty((len(conds), 4, 2), dtype=torch.int64, device="cuda")
    miss = torch.zeros(1, dtype=torch.int64, device="cuda")
    olap.text_ranges_device(dg, ext, len(conds), torch.from_numpy(kinds).cuda(), torch.from_numpy(first).cuda(), None,
                            torch.from_numpy(buf.copy()).cuda(), torch.from_numpy(offs).cuda(), len(offs) - 1, out, miss)
    torch.cuda.synchronize()
    assert np.array_equal(out.cpu().numpy(), want) and int(miss.item()) == wmiss


# ------------------------------------------------------------------ fact-table partitions (NEXT #4, Fig. 7)

def _check_table(got, ref, cols, qs):
    ops = np.array([q[2] for q in qs], np.int32)
    isf = np.array([cols[q[1]].dtype == np.float32 for q in qs])
    assert np.array_equal(got["flags"], ref["flags"]) and np.array_equal(got["i"], ref["i"])
    ex = ~isf | (ops == olap.MIN) | (ops == olap.MAX) | (ops == olap.COUNT)
    assert np.array_equal(got["d"][ex], ref["d"][ex])
    tol = 1e-6 * np.abs(ref["d"]) + 1e-300
    assert (np.abs(got["d"] - ref["d"]) <= tol).all()


def _dev_table_queries(qs):
    off, ca, dcol, ops = olap.pack_table_queries(qs)
    return [torch.from_numpy(a.view(np.uint8) if a.dtype.names else a).cuda() for a in (off, ca, dcol, ops)]


@pytest.mark.parametrize("sm_count", [1, 2, 4, 37, 0])
def test_table_partition_parity(sm_count):
    """A partition of 1/2/4 SMs (the paper's Fig. 7 sizes), an odd count and the whole GPU:
    same answers as the oracle, grid bounded by the partition."""
    nrows = 200_003
    rng = np.random.default_rng(sm_count + 100)
    cols = _table_cols(nrows, rng)
    t = olap.Table(nrows, [c.dtype for c in cols])
    for i, c in enumerate(cols):
        t.load_column(i, c)
    p = olap.TablePart(t, sm_count)
    nsm = torch.cuda.get_device_properties(0).multi_processor_count
    assert p.sm_count == (sm_count if 0 < sm_count <= nsm else nsm)
    assert 1 <= p.blocks and p.blocks % p.sm_count == 0
    qs = _table_queries(rng, 300)
    qs.append(([], 5, olap.SUM))
    qs.append(([(1, 3, 3), (1, 4, 4)], 4, olap.MIN))        # contradictory -> empty
    qs.append(([(0, 0, 39)], 1, olap.COUNT))                 # every query COUNT-free columns mix
    d = _dev_table_queries(qs)
    res = torch.empty(len(qs) * olap.RESULT_DTYPE.itemsize, dtype=torch.uint8, device="cuda")
    p.query_device(len(qs), *d, res)
    torch.cuda.synchronize()
    got = res.cpu().numpy().view(olap.RESULT_DTYPE)
    _check_table(got, oracle.tablescan(cols, qs, nthreads=oracle.max_threads()), cols, qs)


def test_table_partitions_concurrent_streams():
    """Six partitions of 1/1/2/2/4/4 SMs (Fig. 7) on one table, each on its own stream,
    launched back to back: every batch equals the oracle (own workspaces, no sharing)."""
    nrows = 100_000
    rng = np.random.default_rng(7)
    cols = _table_cols(nrows, rng)
    t = olap.Table(nrows, [c.dtype for c in cols])
    for i, c in enumerate(cols):
        t.load_column(i, c)
    parts = [olap.TablePart(t, s) for s in (1, 1, 2, 2, 4, 4)]
    streams = [torch.cuda.Stream() for _ in parts]
    batches, outs = [], []
    for p, s in zip(parts, streams):
        qs = _table_queries(rng, int(rng.integers(1, 120)))
        d = _dev_table_queries(qs)
        res = torch.empty(len(qs) * olap.RESULT_DTYPE.itemsize, dtype=torch.uint8, device="cuda")
        torch.cuda.current_stream().synchronize()
        with torch.cuda.stream(s):
            p.query_device(len(qs), *d, res, stream=s)
        batches.append((qs, d))
        outs.append(res)
    torch.cuda.synchronize()
    for (qs, _d), res in zip(batches, outs):
        got = res.cpu().numpy().view(olap.RESULT_DTYPE)
        _check_table(got, oracle.tablescan(cols, qs, nthreads=oracle.max_threads()), cols, qs)


def test_table_partition_boxes():
    """Box-form queries over dimension columns (e.g. olap_text_ranges output): a full-range
    dimension is no condition, an empty range matches nothing; equal to the oracle on the
    equivalent condition lists."""
    nrows = 150_001
    rng = np.random.default_rng(3)
    cols = _table_cols(nrows, rng)
    ext = (40, 7, 13, 5)
    t = olap.Table(nrows, [c.dtype for c in cols])
    for i, c in enumerate(cols):
        t.load_column(i, c)
    p = olap.TablePart(t, 4)
    nq = 400
    lo = np.zeros((nq, 4), np.int64)
    hi = np.zeros((nq, 4), np.int64)
    for q in range(nq):
        for d, n in enumerate(ext):
            r = rng.random()
            if r < 0.4:
                lo[q, d], hi[q, d] = 0, n - 1                     # full: no condition
            elif r < 0.45:
                lo[q, d], hi[q, d] = 1, 0                         # empty
            else:
                a, b = sorted(rng.integers(0, n, size=2))
                lo[q, d], hi[q, d] = a, b
    dcol = rng.integers(4, 6, size=nq).astype(np.int32)
    ops = rng.integers(0, 5, size=nq).astype(np.int32)
    flat = np.stack([lo, hi], axis=-1).reshape(-1)                # olap_range {lo, hi} query-major
    qs = []
    for q in range(nq):
        conds = [(d, int(lo[q, d]), int(hi[q, d])) for d in range(4)
                 if not (lo[q, d] == 0 and hi[q, d] == ext[d] - 1)]
        qs.append((conds, int(dcol[q]), int(ops[q])))
    res = torch.empty(nq * olap.RESULT_DTYPE.itemsize, dtype=torch.uint8, device="cuda")
    p.query_boxes_device(nq, [0, 1, 2, 3], ext, torch.from_numpy(flat).cuda(), torch.from_numpy(dcol).cuda(),
                         torch.from_numpy(ops).cuda(), res)
    torch.cuda.synchronize()
    got = res.cpu().numpy().view(olap.RESULT_DTYPE)
    _check_table(got, oracle.tablescan(cols, qs, nthreads=oracle.max_threads()), cols, qs)


@pytest.mark.parametrize("dtype", [np.int32, np.float32])
@pytest.mark.parametrize("ext", [(64, 129, 7), (8, 8, 16, 16, 16, 16), (3, 1000), (2, 9, 16384), (40, 1024, 1024)])
def test_warp_items_large_batches(ext, dtype):
    """Batches of more than 8 queries per resident block take warp-granular items
    (reduce_kernel_w): same bars as the block-item path, deterministic."""
    n = int(np.prod(ext))
    seed = 0x5EED5000 + n
    rng = np.random.default_rng(seed)
    boxes = np.concatenate([synth.random_boxes(ext, 2000, rng), synth.fraction_boxes(ext, 2000, rng, 1e-4),
                            synth.small_boxes(ext, 4000, rng, bytes_lo=4, bytes_hi=1 << 16)])
    ops = synth.ops_uniform(len(boxes), rng)
    c = olap.Cube(ext, dtype)
    c.fill(olap.GEN_UNIFORM, seed)
    got = c.query(boxes, ops)
    idx = np.arange(len(boxes)) if n <= (1 << 22) else rng.choice(len(boxes), 600, replace=False)
    ref = oracle.query(ext, boxes[idx], ops[idx], dtype=dtype, gen=oracle.GEN_UNIFORM, seed=seed,
                       nthreads=oracle.max_threads())
    compare(got[idx], ref, ops[idx], dtype)
    assert np.array_equal(c.query(boxes, ops), got)


def test_host_batches_replay_cuda_graphs(monkeypatch):
    """olap_query_batch replays a per-batch-size CUDA graph for batches of
    <= 16,384 queries.  Replays equal the direct path bit for bit, across sizes (LRU of four
    graphs), after a workspace growth (graphs invalidated), on a bricked cube, and interleaved
    with device batches on another stream."""
    for ext, layout in (((32, 32, 32, 32), olap.LAYOUT_ROWMAJOR), ((16, 96, 136), olap.LAYOUT_BRICK),
                        ((64, 16, 16, 16, 192), olap.LAYOUT_ROWMAJOR)):
        c = olap.Cube(ext, np.float32, layout=layout)
        c.fill(olap.GEN_UNIFORM, 9)
        rng = np.random.default_rng(9)
        sizes = [1000, 17, 1000, 3000, 5, 999, 1000, 20000, 1000]
        batches = {n: (synth.fraction_boxes(ext, n, rng, 1e-4), synth.ops_uniform(n, rng)) for n in set(sizes)}
        monkeypatch.setenv("OLAP_NO_GRAPHS", "1")
        ref = {n: c.query(*batches[n]) for n in batches}
        monkeypatch.delenv("OLAP_NO_GRAPHS")
        k0 = c.stats()[0]
        for i, n in enumerate(sizes):
            got = c.query(*batches[n])
            assert got.tobytes() == ref[n].tobytes(), (ext, n, i)
            if i == 4:  # a device batch on another stream between host batches
                b, o = batches[1000]
                res = torch.empty(1000 * 24, dtype=torch.uint8, device="cuda")
                s = torch.cuda.Stream()
                c.query_device(torch.from_numpy(b).cuda(), torch.from_numpy(o).cuda(), res, stream=s)
                s.synchronize()
                assert res.cpu().numpy().tobytes() == ref[1000].tobytes()
        assert c.stats()[0] > k0  # replayed kernels are counted
        idx = np.arange(0, 1000, 37)
        b, o = batches[1000]
        want = oracle.query(ext, b[idx], o[idx], dtype=np.float32, gen=oracle.GEN_UNIFORM, seed=9,
                            nthreads=oracle.max_threads())
        compare(ref[1000][idx], want, o[idx], np.float32)
