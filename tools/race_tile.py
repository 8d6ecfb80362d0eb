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
