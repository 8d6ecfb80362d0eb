"""N>1 host path on CPU: world_size-2 gloo process groups.

1. The exchange algebra.  Each rank owns a block-cyclic dim-0 shard of the cube
   (olap_shard_local_rows from the product's C-ABI gives its local row range), computes its
   partials over its local box (here with the oracle on the shard's rows, since kernels need a
   GPU), encodes them in the olap.h partial format, and the two element-wise reductions the
   library's NCCL exchange performs (mgpu.cu: ncclSum on the sums as uint64 / float64, ncclMax
   on the int32 codes) are applied across the ranks with gloo all-reduces of the same types.
   The decoded result must equal the oracle on the global cube.
2. The communicator bootstrap of dist.py: rank 0's olap_comm_unique_id reaches every rank
   through the process group, and olap_comm_init_rank without a GPU fails loudly (E_CUDA).
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import synth

INT_MIN = -(2 ** 31)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _code(v, dtype):
    if dtype == np.int32:
        return np.int32(v)
    b = np.array([v], np.float32).view(np.int32)[0]
    return np.int32(b ^ ((b >> 31) & 0x7FFFFFFF))


def _decode(c, dtype):
    if dtype == np.int32:
        return int(c)
    b = np.int32(c ^ ((c >> 31) & 0x7FFFFFFF))
    return float(np.array([b], np.int32).view(np.float32)[0])


def _worker(rank, world, port, dtype_name, block, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_ipps_malikrse12_b200 as olap

        dtype = np.dtype(dtype_name)
        ext = (23, 6, 9)
        cells = synth.uniform_cells(int(np.prod(ext)), dtype, 0x5EED3000).reshape(ext)
        rng = np.random.default_rng(17)
        boxes = synth.random_boxes(ext, 200, rng)
        ops = synth.ops_uniform(200, rng)
        ops[ops == oracle.COUNT] = oracle.SUM
        owned = [r for r in range(ext[0]) if (r // block) % world == rank]
        local = cells[owned]                              # local rows in local order
        nq = len(boxes)
        psum = torch.zeros(nq, dtype=torch.int64)
        pext = torch.full((2 * nq,), INT_MIN, dtype=torch.int32)
        lb = boxes.copy()
        for i in range(nq):
            llo, lhi = olap.shard_local_rows(ext[0], (world, rank, block), int(boxes[i, 0, 0]), int(boxes[i, 0, 1]))
            if llo > lhi:
                continue
            lb[i, 0] = (llo, lhi)
            r = oracle.query((len(owned),) + ext[1:], lb[i:i + 1], [oracle.SUM], local.ravel())
            mn = oracle.query((len(owned),) + ext[1:], lb[i:i + 1], [oracle.MIN], local.ravel())
            mx = oracle.query((len(owned),) + ext[1:], lb[i:i + 1], [oracle.MAX], local.ravel())
            if dtype == np.int32:
                psum[i] = int(r["i"][0])
                pext[2 * i] = int(_code(mx["i"][0], dtype))
                pext[2 * i + 1] = int(~_code(mn["i"][0], dtype))
            else:
                psum[i] = int(np.array([r["d"][0]], np.float64).view(np.int64)[0])
                pext[2 * i] = int(_code(mx["d"][0], dtype))
                pext[2 * i + 1] = int(~_code(mn["d"][0], dtype))
        code = olap.INT32 if dtype == np.int32 else olap.FLOAT32
        # the library's exchange (mgpu.cu): ncclSum on uint64 (int32 cube, wraparound) or
        # float64 sums, ncclMax on the int32 codes -- the same reductions over gloo
        if code == olap.FLOAT32:
            dist.all_reduce(psum.view(torch.float64), op=dist.ReduceOp.SUM)
        else:
            dist.all_reduce(psum, op=dist.ReduceOp.SUM)
        dist.all_reduce(pext, op=dist.ReduceOp.MAX)
        ref = oracle.query(ext, boxes, ops, cells.ravel())
        bad = 0
        for i in range(nq):
            if ops[i] == oracle.SUM or ops[i] == oracle.AVG:
                if dtype == np.int32:
                    s = int(psum[i])
                    got = s if ops[i] == oracle.SUM else s / float(np.prod(boxes[i, :, 1] - boxes[i, :, 0] + 1))
                    want = ref["i"][i] if ops[i] == oracle.SUM else ref["d"][i]
                    bad += got != want
                else:
                    s = float(np.array([int(psum[i])], np.int64).view(np.float64)[0])
                    V = float(np.prod(boxes[i, :, 1] - boxes[i, :, 0] + 1))
                    got = s if ops[i] == oracle.SUM else s / V
                    bad += abs(got - ref["d"][i]) > 1e-12 * abs(ref["d"][i])
            elif ops[i] == oracle.MAX:
                want = ref["i"][i] if dtype == np.int32 else ref["d"][i]
                bad += _decode(np.int32(pext[2 * i]), dtype) != want
            elif ops[i] == oracle.MIN:
                want = ref["i"][i] if dtype == np.int32 else ref["d"][i]
                bad += _decode(np.int32(~np.int32(pext[2 * i + 1])), dtype) != want
        q.put((rank, int(bad)))
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put((rank, repr(e)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("dtype_name,block", [("int32", 1), ("float32", 1), ("int32", 3), ("float32", 4)])
def test_two_rank_exchange_equals_oracle(dtype_name, block):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, dtype_name, block, q)) for r in range(2)]
    for p in procs:
        p.start()
    out = [q.get(timeout=180) for _ in procs]
    for p in procs:
        p.join(timeout=60)
    for rank, bad in out:
        assert bad == 0, f"rank {rank}: {bad}"


def _boot_worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_ipps_malikrse12_b200 as olap
        from paper_conf_ipps_malikrse12_b200.dist import broadcast_comm_id

        uid = broadcast_comm_id(rank)
        got = [None] * world
        dist.all_gather_object(got, uid)
        status = None
        if not torch.cuda.is_available():
            try:
                olap.Comm(uid, world, rank, 0)
            except olap.OlapError as e:
                status = e.status
        q.put((rank, len(uid), all(g == got[0] for g in got), status))
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put((rank, repr(e), False, None))
    finally:
        dist.destroy_process_group()


def test_two_rank_comm_id_bootstrap():
    """dist.broadcast_comm_id: every rank receives rank 0's 128-byte communicator id."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_boot_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    out = [q.get(timeout=180) for _ in procs]
    for p in procs:
        p.join(timeout=60)
    import paper_conf_ipps_malikrse12_b200 as olap
    for rank, n, same, status in out:
        assert n == 128 and same, (rank, n, same)
        if not torch.cuda.is_available():
            assert status == olap.E_CUDA, status
