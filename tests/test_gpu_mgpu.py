"""GPU parity of the sharded path with the exchange inside the library.

gpurun gives one B200, so the multi-GPU code paths run on cuda:0:
  * group handles (olap_cube_create_multi) with G = 1 x shards_per_device shards on device 0:
    the shards reduce, fold on the device in shard order, and the partials go through a
    1-rank NCCL communicator (ncclCommInitAll + ncclReduce) before the finalize;
  * a shard with an attached 1-rank communicator (olap_comm_init_rank + ncclAllReduce, the
    one-process-per-GPU path of bench.py --gpus N);
  * olap_query_stream's pipelined batches (exchange of batch k overlapping batch k+1).
Every answer is compared with the oracle on the GLOBAL cube (int32 bit-exact; float32 within
1e-6 of the fp64 oracle).
"""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_ipps_malikrse12_b200 as olap
import synth
from test_gpu_parity import compare

pytestmark = pytest.mark.gpu


def _batch(ext, n, seed):
    rng = np.random.default_rng(seed)
    boxes = np.concatenate([synth.random_boxes(ext, n // 2, rng), synth.fraction_boxes(ext, n - n // 2, rng, 1e-4)])
    ops = synth.ops_uniform(len(boxes), rng)
    boxes[3, 1] = [4, 2]  # lo > hi: EMPTY
    return boxes, ops


def _ref(ext, boxes, ops, dtype, seed):
    return oracle.query(ext, boxes, ops, dtype=dtype, gen=oracle.GEN_UNIFORM, seed=seed, nthreads=oracle.max_threads())


@pytest.mark.parametrize("spd,block", [(1, 1), (2, 1), (3, 2), (4, 1), (8, 3)])
@pytest.mark.parametrize("dtype", [np.int32, np.float32])
def test_group_handle_equals_oracle(spd, block, dtype):
    ext = (37, 12, 10, 66)
    seed = 0x5EED7000 + spd
    c = olap.Cube(ext, dtype, devices=[0], shards_per_device=spd, shard_block=block)
    c.fill(olap.GEN_UNIFORM, seed)
    rows, cells, ptr = c.info()
    assert rows == ext[0] and ptr is None
    boxes, ops = _batch(ext, 600, seed)
    ref = _ref(ext, boxes, ops, dtype, seed)
    compare(c.query(boxes, ops), ref, ops, dtype)
    # device-buffer path on devices[0]
    res = torch.empty(len(ops) * olap.RESULT_DTYPE.itemsize, dtype=torch.uint8, device="cuda")
    s = torch.cuda.Stream()
    c.query_device(torch.from_numpy(boxes).cuda(), torch.from_numpy(ops).cuda(), res, stream=s)
    s.synchronize()
    compare(res.cpu().numpy().view(olap.RESULT_DTYPE), ref, ops, dtype)
    # pipelined stream in ragged batches
    for batch in (1, 37, 256, 0):
        compare(c.query_stream(boxes[:300], ops[:300], batch=batch), ref[:300], ops[:300], dtype)
    n, _ = c.stats()
    assert n > 0


def test_group_handle_deterministic_and_load():
    """Float sums across shards fold in a fixed order: bit-identical run to run; load() of a host
    cube distributes rows to the shards."""
    ext = (21, 40, 33)
    cells = synth.uniform_cells(int(np.prod(ext)), np.float32, 99) * np.float32(3.0) - np.float32(1.5)
    c = olap.Cube(ext, np.float32, devices=[0], shards_per_device=5, shard_block=2)
    c.load(cells)
    boxes, ops = _batch(ext, 500, 5)
    a = c.query(boxes, ops)
    b = c.query_stream(boxes, ops, batch=64)
    assert a.tobytes() == b.tobytes()
    ref = oracle.query(ext, boxes, ops, cells)
    # signed non-integer cells: |gpu - oracle| <= 1e-6 * sum|x| (reading S8's mixed-sign bar)
    absref = oracle.query(ext, boxes, np.where(ops == oracle.AVG, oracle.SUM, ops).astype(np.int32), np.abs(cells))
    sums = (ops == oracle.SUM) | (ops == oracle.AVG)
    assert np.array_equal(a["flags"], ref["flags"])
    ex = ~sums
    assert np.array_equal(a["d"][ex], ref["d"][ex]) and np.array_equal(a["i"], ref["i"])
    V = np.prod(boxes[:, :, 1] - boxes[:, :, 0] + 1, axis=1).astype(np.float64)
    bound = 1e-6 * np.where(ops == oracle.AVG, absref["d"] / np.maximum(V, 1), absref["d"])
    assert np.all(np.abs(a["d"][sums] - ref["d"][sums]) <= bound[sums] + 1e-300)


def test_group_handle_bricked_and_large():
    """A bricked group (C5's layout) and a group over a cube that takes the tile path."""
    ext = (16, 96, 136)
    c = olap.Cube(ext, np.int32, devices=[0], shards_per_device=3, layout=olap.LAYOUT_BRICK)
    c.fill(olap.GEN_UNIFORM, 13)
    b, o = synth.config_queries("C5", nq=400, seed=3, extents=ext)
    compare(c.query(b, o), _ref(ext, b, o, np.int32, 13), o, np.int32)
    big = (64, 16, 16, 16, 192)  # 192 MiB: every shard > 64 MiB takes the L2 order / tile planner
    g = olap.Cube(big, np.float32, devices=[0], shards_per_device=2)
    g.fill(olap.GEN_UNIFORM, 11)
    rng = np.random.default_rng(4)
    tb = synth.fraction_boxes(big, 256, rng, 1e-2, 0.5)
    to = synth.ops_mix(256, rng)
    got = g.query_stream(tb, to, batch=128)
    assert g.tile_stats()[3], "the shards' batches should take the tile-shared scan"
    compare(got, _ref(big, tb, to, np.float32, 11), to, np.float32)


def test_attached_comm_one_rank():
    """One process per GPU (bench.py --gpus N): a 1-rank library communicator attached to a
    {1, 0, 1} shard; host, device and stream paths, plus the exchange entry point alone."""
    ext = (30, 17, 129)
    seed = 0x5EED7100
    comm = olap.Comm(olap.comm_unique_id(), 1, 0, 0)
    c = olap.Cube(ext, np.int32, shard=(1, 0, 1))
    c.fill(olap.GEN_UNIFORM, seed)
    c.attach_comm(comm)
    boxes, ops = _batch(ext, 700, seed)
    ref = _ref(ext, boxes, ops, np.int32, seed)
    compare(c.query(boxes, ops), ref, ops, np.int32)
    compare(c.query_stream(boxes, ops, batch=100), ref, ops, np.int32)
    res = torch.empty(len(ops) * olap.RESULT_DTYPE.itemsize, dtype=torch.uint8, device="cuda")
    c.query_device(torch.from_numpy(boxes).cuda(), torch.from_numpy(ops).cuda(), res)
    torch.cuda.synchronize()
    compare(res.cpu().numpy().view(olap.RESULT_DTYPE), ref, ops, np.int32)
    comm.check()
    # exchange alone on a 1-rank communicator is the identity
    s = torch.arange(50, dtype=torch.int64, device="cuda") - 20
    e = torch.arange(100, dtype=torch.int32, device="cuda") - 7
    s0, e0 = s.clone(), e.clone()
    olap.exchange_partials_device(comm, np.int32, 50, s, e)
    torch.cuda.synchronize()
    assert torch.equal(s, s0) and torch.equal(e, e0)
    c.attach_comm(None)  # detached: a {1, 0, 1} shard is the whole cube, answered without NCCL
    compare(c.query(boxes, ops), ref, ops, np.int32)
    c.close()
    comm.close()
    assert olap.nccl_version() >= 21800


def test_multi_errors():
    with pytest.raises(olap.OlapError) as ei:
        olap.Cube((8, 8), np.int32, devices=[0, 0])
    assert ei.value.status == olap.E_INVALID
    g = olap.Cube((8, 8), np.int32, devices=[0], shards_per_device=2)
    d = torch.zeros(16, dtype=torch.int64, device="cuda")
    with pytest.raises(olap.OlapError) as ei:
        g.partials_device(torch.zeros((1, 2, 2), dtype=torch.int64, device="cuda"),
                          torch.zeros(1, dtype=torch.int32, device="cuda"), d, d.view(torch.int32))
    assert ei.value.status == olap.E_UNSUPPORTED
    with pytest.raises(olap.OlapError) as ei:
        g.query(np.array([[[0, 8], [0, 1]]]), np.array([0], np.int32))
    assert ei.value.status == olap.E_RANGE
    sh = olap.Cube((8, 8), np.int32, shard=(2, 1, 1))
    with pytest.raises(olap.OlapError) as ei:
        sh.query(np.array([[[0, 3], [0, 1]]]), np.array([0], np.int32))
    assert ei.value.status == olap.E_STATE
    comm = olap.Comm(olap.comm_unique_id(), 1, 0, 0)
    with pytest.raises(olap.OlapError) as ei:
        sh.attach_comm(comm)  # shard 1 of 2 vs rank 0 of 1
    assert ei.value.status == olap.E_INVALID
    comm.close()


def test_group_handle_invalid_growth_and_stream_errors():
    """Device batches flag out-of-range queries INVALID (the host path fails the whole batch with
    E_RANGE naming the query); the executor's buffers grow across calls; a stream with a bad query
    fails as a whole and leaves the cube usable."""
    ext = (24, 9, 70)
    seed = 0x5EED7200
    c = olap.Cube(ext, np.float32, devices=[0], shards_per_device=3, shard_block=2)
    c.fill(olap.GEN_UNIFORM, seed)
    for n in (10, 1500, 5000, 300):  # growth past the first capacity, then a smaller batch again
        boxes, ops = _batch(ext, n, seed + n)
        compare(c.query(boxes, ops), _ref(ext, boxes, ops, np.float32, seed), ops, np.float32)
    boxes, ops = _batch(ext, 200, seed + 1)
    bad = boxes.copy()
    bad[7, 2] = [5, 70]  # hi == extent: out of range
    res = torch.empty(200 * olap.RESULT_DTYPE.itemsize, dtype=torch.uint8, device="cuda")
    c.query_device(torch.from_numpy(bad).cuda(), torch.from_numpy(ops).cuda(), res)
    torch.cuda.synchronize()
    got = res.cpu().numpy().view(olap.RESULT_DTYPE)
    assert got["flags"][7] == olap.RESULT_INVALID
    ok = np.arange(200) != 7
    compare(got[ok], _ref(ext, boxes[ok], ops[ok], np.float32, seed), ops[ok], np.float32)
    with pytest.raises(olap.OlapError) as ei:
        c.query(bad, ops)
    assert ei.value.status == olap.E_RANGE and "query 7" in str(ei.value)
    with pytest.raises(olap.OlapError) as ei:
        c.query_stream(bad, ops, batch=64)
    assert ei.value.status == olap.E_RANGE
    compare(c.query_stream(boxes, ops, batch=64), _ref(ext, boxes, ops, np.float32, seed), ops, np.float32)


def test_plain_cube_stream_equals_batches():
    """olap_query_stream on a plain cube (no exchange): pipelined copy-in / reduce / copy-out in
    batches of any size equals olap_query_batch on the whole, bit for bit (int32)."""
    ext = (40, 33, 17)
    c = olap.Cube(ext, np.int32)
    c.fill(olap.GEN_UNIFORM, 77)
    boxes, ops = _batch(ext, 3000, 77)
    want = c.query(boxes, ops)
    for batch in (1, 999, 1024, 2999, 3000, 0):
        assert c.query_stream(boxes, ops, batch=batch).tobytes() == want.tobytes(), batch
    compare(want, _ref(ext, boxes, ops, np.int32, 77), ops, np.int32)
