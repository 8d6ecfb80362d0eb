"""compute-sanitizer target: one small batch through the tile-shared scan (slot trees, column mode,
edge cells) and one through the item path, checked against the oracle.  Usage (GPU box):
compute-sanitizer --tool racecheck python tools/race_tile.py"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
import paper_conf_ipps_malikrse12_b200 as olap  # noqa: E402
import synth  # noqa: E402

ext = (32, 16, 16, 16, 192)  # 96 MiB: the tile path is enabled (> 64 MiB)
c = olap.Cube(ext, np.float32)
c.fill(olap.GEN_UNIFORM, 5)
rng = np.random.default_rng(5)
b = np.concatenate([synth.fraction_boxes(ext, 64, rng, 1e-2, 0.5), np.array([[[0, e - 1] for e in ext]])])
o = synth.ops_uniform(len(b), rng)
got = c.query(b, o)
assert c.tile_stats()[3], "expected the tile path"
ref = oracle.query(ext, b, o, dtype=np.float32, gen=oracle.GEN_UNIFORM, seed=5, nthreads=oracle.max_threads())
ok = np.array_equal(got["flags"], ref["flags"]) and np.allclose(got["d"], ref["d"], rtol=1e-6, atol=0)
print("tile path", "ok" if ok else "MISMATCH")

# row-aligned runs (256-cell rows): the per-query pattern loop over the transposed slot trees,
# 64-KiB float tiles; and an int32 cube (48-KiB tiles, int64 tree entries)
for ext2, dt, seed in (((32, 16, 16, 16, 256), np.float32, 6), ((32, 16, 16, 16, 256), np.int32, 7)):
    c2 = olap.Cube(ext2, dt)
    c2.fill(olap.GEN_UNIFORM, seed)
    rng2 = np.random.default_rng(seed)
    b2 = synth.fraction_boxes(ext2, 48, rng2, 1e-2, 0.5)
    o2 = synth.ops_uniform(len(b2), rng2)
    got2 = c2.query(b2, o2)
    assert c2.tile_stats()[3], "expected the tile path"
    ref2 = oracle.query(ext2, b2, o2, dtype=dt, gen=oracle.GEN_UNIFORM, seed=seed, nthreads=oracle.max_threads())
    ok2 = np.array_equal(got2["flags"], ref2["flags"]) and np.array_equal(got2["i"], ref2["i"]) and \
        np.allclose(got2["d"], ref2["d"], rtol=1e-6, atol=0)
    print("tile pattern path", np.dtype(dt).name, "ok" if ok2 else "MISMATCH")
    c2.close()

# 2 x 4 x 4-bricked cube (brick_reduce_kernel<., ., 1>) and a fact-table scan (query-chunked blocks)
kb = (10, 96, 136)
k3 = olap.Cube(kb, np.int32, layout=olap.LAYOUT_BRICK3)
k3.fill(olap.GEN_UNIFORM, 13)
sb, so = synth.config_queries("C5", nq=256, seed=3, extents=kb)
refb = oracle.query(kb, sb, so, dtype=np.int32, gen=oracle.GEN_UNIFORM, seed=13)
print("brick3", "ok" if k3.query(sb, so).tobytes() == refb.tobytes() else "MISMATCH")
nrows = 5000
trng = np.random.default_rng(9)
cols = [trng.integers(0, n, size=nrows).astype(np.int32) for n in (40, 7, 13)] + [trng.random(nrows).astype(np.float32)]
t = olap.Table(nrows, [x.dtype for x in cols])
for i, x in enumerate(cols):
    t.load_column(i, x)
qs = [([(0, int(a), int(a) + 5), (1, 2, 4)], 3, int(op)) for a, op in zip(trng.integers(0, 35, 300), trng.integers(0, 5, 300))]
gt = t.query(qs)
rt = oracle.tablescan(cols, qs)
print("table", "ok" if np.array_equal(gt["flags"], rt["flags"]) and np.allclose(gt["d"], rt["d"], rtol=1e-6) else "MISMATCH")
