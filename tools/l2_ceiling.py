"""Dev experiment: reduce-kernel throughput when the cube is L2-resident (upper bound for
an L2-reuse schedule).  C2a recipe on a (1,16,16,16,16,256) = 64 MiB float32 cube."""
import json
import sys
import os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_ipps_malikrse12_b200 as olap
import synth

for ext in [(1, 16, 16, 16, 16, 256), (2, 16, 16, 16, 16, 256), (16, 16, 16, 16, 16, 256)]:
    c = olap.Cube(ext, np.float32)
    c.fill(olap.GEN_UNIFORM, 1)
    bs = [synth.config_queries("C2a", nq=4096, seed=100 + k, extents=ext) for k in range(8)]
    dev = [(torch.from_numpy(b).cuda(), torch.from_numpy(o).cuda()) for b, o in bs]
    res = torch.empty(4096 * 24, dtype=torch.uint8, device="cuda")
    st = torch.cuda.Stream()
    for k in range(3):
        c.query_device(*dev[k], res, stream=st)
    st.synchronize()
    c.profile(True)
    for k in range(3, 8):
        c.query_device(*dev[k], res, stream=st)
    st.synchronize()
    ms, n, b = c.profile_read()
    print(json.dumps({"extents": ext, "cube_mib": int(np.prod(ext)) * 4 >> 20, "reduce_ms_per_launch": ms / n,
                      "alg_GBps": b / (ms / 1e3) / 1e9}))
    c.close()
