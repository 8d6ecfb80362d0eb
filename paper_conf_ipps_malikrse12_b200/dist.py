"""One process per GPU: the sharded cube on a torch.distributed job.

Rank g holds shard g of a block-cyclic dim-0 split of the global cube.  The whole query path
(shard-local plan + range-reduce, the NCCL exchange of the per-query partials, the finalize) runs
inside the library: this module only bootstraps the library's NCCL communicator — rank 0 asks the
library for a communicator id (olap_comm_unique_id) and torch.distributed broadcasts its 128
bytes — and attaches it to the rank's shard (olap_cube_attach_comm).  torch.distributed is the
out-of-band channel, nothing more; no partial crosses it.
"""
from __future__ import annotations

import numpy as np

from . import RESULT_DTYPE, Comm, Cube, comm_unique_id


def broadcast_comm_id(rank: int, group=None) -> bytes:
    """Rank 0's olap_comm_unique_id, broadcast to every rank of `group` (any backend)."""
    import torch.distributed as dist

    box = [comm_unique_id() if rank == 0 else None]
    dist.broadcast_object_list(box, src=0, group=group)
    uid = box[0]
    if not isinstance(uid, (bytes, bytearray)) or len(uid) != 128:
        raise RuntimeError("communicator id broadcast failed")
    return bytes(uid)


def init_comm(rank: int, world: int, device: int, group=None) -> Comm:
    """The library's NCCL communicator for this rank (collective over the process group)."""
    return Comm(broadcast_comm_id(rank, group), world, rank, device)


class ShardedCube:
    """This rank's shard of a cube sharded over the default process group, answering batches
    as collectives through the library (olap_query_batch / _device / olap_query_stream)."""

    def __init__(self, extents, dtype, rank: int, world: int, block: int = 1, device: int = 0, group=None,
                 layout: int = 0, comm: Comm | None = None):
        self.extents = tuple(int(e) for e in extents)
        self.cube = Cube(self.extents, dtype, shard=(world, rank, block), device=device, layout=layout)
        self.dtype_code = self.cube.dtype_code
        self.rank, self.world = rank, world
        self.comm = comm if comm is not None else init_comm(rank, world, device, group)
        self.cube.attach_comm(self.comm)

    def fill(self, *a, **k):
        self.cube.fill(*a, **k)

    def query_device(self, d_ranges, d_ops, d_results, nq: int | None = None, stream=None):
        self.cube.query_device(d_ranges, d_ops, d_results, nq=nq, stream=stream)

    def query(self, ranges, ops, out: np.ndarray | None = None) -> np.ndarray:
        """Host arrays in, host results out (every rank gets every answer)."""
        return self.cube.query(ranges, ops, out=out)

    def query_stream(self, ranges, ops, batch: int = 0) -> np.ndarray:
        return self.cube.query_stream(ranges, ops, batch=batch)

    def close(self):
        self.cube.attach_comm(None)
        self.cube.close()
        self.comm.close()


__all__ = ["broadcast_comm_id", "init_comm", "ShardedCube", "RESULT_DTYPE"]
