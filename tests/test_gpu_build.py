"""NEXT #2 on the GPU ("building the cube from relational tables",
PAPER.md:252/450 "every text column is converted to integer column"):
  * bulk encoding: a fact table's raw string columns (millions of rows) translated on the GPU
    (olap_dict_translate_device) equal the oracle's std::map ids, bit for bit;
  * deterministic float32 cube build (olap_cube_add_facts_device: sort by cell, fp64 per cell
    in row order, one rounding) equals oracle.factbuild bit for bit and is identical run to run,
    also on a shard; int32 builds stay exact.
"""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_ipps_malikrse12_b200 as olap
import synth

pytestmark = pytest.mark.gpu


def test_bulk_encoding_of_fact_text_columns():
    members = synth.tpcds_members()
    nrows = 1 << 22
    facts, _, _ = synth.tpcds_facts(nrows, members)
    for col in ("ca_state", "i_class", "s_store_id", "d_date"):
        d = olap.Dict(members[col])
        od = oracle.Dict(members[col])
        raw, offs = synth.text_column(members[col], facts[col])
        d_ids = torch.empty(nrows, dtype=torch.int32, device="cuda")
        miss = torch.zeros(1, dtype=torch.int64, device="cuda")
        olap.translate_device([d], None, torch.from_numpy(raw).cuda(), torch.from_numpy(offs).cuda(), nrows, d_ids,
                              miss)
        torch.cuda.synchronize()
        got = d_ids.cpu().numpy()
        assert int(miss.item()) == 0
        # the oracle on the raw row strings themselves (first 200k rows) ...
        n = 200_000
        keys = [bytes(raw[offs[i]:offs[i + 1]]) for i in range(n)]
        assert np.array_equal(got[:n], od.translate(keys))
        # ... and on every row through its member (identical strings, identical ids)
        assert np.array_equal(got, od.translate(members[col])[facts[col]])


def _cells_of(c, ext, dtype, shard=None):
    """Every cell of a (shard of a) cube through 1-cell MAX partials (exact value, any dtype)."""
    boxes = np.stack(np.meshgrid(*[np.arange(n) for n in ext], indexing="ij"), -1).reshape(-1, len(ext))
    boxes = np.repeat(boxes[:, :, None], 2, axis=2)
    nq = len(boxes)
    s = torch.empty(nq, dtype=torch.int64, device="cuda")
    e = torch.empty(2 * nq, dtype=torch.int32, device="cuda")
    c.partials_device(torch.from_numpy(boxes).cuda(), torch.full((nq,), olap.MAX, dtype=torch.int32, device="cuda"),
                      s, e)
    torch.cuda.synchronize()
    code = e.cpu().numpy()[0::2]
    if dtype == np.float32:
        b = code ^ ((code >> 31) & 0x7FFFFFFF)
        return b.astype(np.int32).view(np.float32)
    return code


@pytest.mark.parametrize("shard", [None, (3, 1, 2)])
def test_float_build_bit_exact_and_deterministic(shard):
    ext = (13, 7, 11)
    rng = np.random.default_rng(21)
    nrows = 300_000  # ~300 rows per cell: the order of the adds matters
    ids = np.stack([rng.integers(0, n, size=nrows) for n in ext]).astype(np.int32)
    ids[1, ::997] = 7       # out of range: skipped
    ids[0, ::1013] = -1
    vals = (rng.standard_normal(nrows) * rng.choice([1e-3, 1.0, 1e3], size=nrows)).astype(np.float32)
    init = rng.standard_normal(ext).astype(np.float32)
    want = oracle.factbuild(ext, ids, vals, init).reshape(ext)
    outs = []
    for _ in range(2):
        c = olap.Cube(ext, np.float32, shard=shard)
        c.load(init)  # a shard copies its own rows of the global host cube
        c.add_facts_device(torch.from_numpy(ids).cuda(), torch.from_numpy(vals).cuda())
        torch.cuda.synchronize()
        outs.append(_cells_of(c, ext, np.float32).reshape(ext))
    assert outs[0].tobytes() == outs[1].tobytes()
    if shard is None:
        assert np.array_equal(outs[0], want)
    else:
        G, g, b = shard
        owned = np.array([(x // b) % G == g for x in range(ext[0])])
        assert np.array_equal(outs[0][owned], want[owned])
        assert np.isnan(outs[0][~owned]).all()  # identity code INT_MIN of rows another shard holds


def test_int32_and_count_build_exact():
    ext = (9, 16, 24)
    rng = np.random.default_rng(22)
    nrows = 400_000
    ids = np.stack([rng.integers(0, n, size=nrows) for n in ext]).astype(np.int32)
    vals = rng.integers(-2 ** 31, 2 ** 31 - 1, size=nrows, dtype=np.int64).astype(np.int32)
    c = olap.Cube(ext, np.int32)
    c.fill(olap.GEN_UNIFORM, 5)
    init = oracle.fill(ext, np.int32, oracle.GEN_UNIFORM, 5)
    c.add_facts_device(torch.from_numpy(ids).cuda(), torch.from_numpy(vals).cuda())
    n = olap.Cube(ext, np.float32)
    n.fill(olap.GEN_AFFINE, 0, np.zeros(4))
    n.add_facts_device(torch.from_numpy(ids).cuda())  # float count cube: +1.0 per row
    torch.cuda.synchronize()
    assert np.array_equal(_cells_of(c, ext, np.int32), oracle.factbuild(ext, ids, vals, init))
    assert np.array_equal(_cells_of(n, ext, np.float32),
                          oracle.factbuild(ext, ids, None, np.zeros(ext, np.float32), dtype=np.float32))
