"""Run a few batches of one bench workload's cube/queries (for ncu captures; no timing).
usage: python tools/prof_batch.py [C2a|C2b|C3|C5] [batches]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import paper_conf_ipps_malikrse12_b200 as olap  # noqa: E402
import synth  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "C2a"
nb = int(sys.argv[2]) if len(sys.argv) > 2 else 2
cfg = synth.CONFIGS[name]
c = olap.Cube(cfg["extents"], np.float32)
c.fill(olap.GEN_UNIFORM, cfg["seed"])
for i in range(nb):
    boxes, ops = synth.config_queries(name, seed=cfg["seed"] + i)
    c.query(boxes, ops)
print(name, "tile stats", c.tile_stats())
