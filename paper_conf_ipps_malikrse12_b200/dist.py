"""Multi-GPU plumbing for the sharded cube.

One process per GPU.  Rank g holds shard g of a block-cyclic dim-0 split of the
global cube.  A batch runs the shard-local plan + range-reduce in the library's
kernels (``olap_query_partials_device``), exchanges the per-query partials with
ONE pair of element-wise all-reduces over NCCL (torch.distributed: SUM on the
int64 / float64 sums, MAX on the order-preserving MIN/MAX codes), then finalizes
in the library's kernel.  The exchange is 16 B per query, latency-bound.
"""
from __future__ import annotations

import numpy as np

from . import FLOAT32, INT32, RESULT_DTYPE, Cube, finalize_device


def exchange_partials(psum, pext, dtype_code: int, group=None):
    """All-reduce partials in place: sums with +, ext codes with max (olap.h partial format).

    Works on CUDA tensors with the nccl backend and on CPU tensors with gloo."""
    import torch
    import torch.distributed as dist

    if dtype_code == FLOAT32:
        dist.all_reduce(psum.view(torch.float64), op=dist.ReduceOp.SUM, group=group)
    else:
        dist.all_reduce(psum, op=dist.ReduceOp.SUM, group=group)   # two's complement wraparound
    dist.all_reduce(pext, op=dist.ReduceOp.MAX, group=group)


class ShardedCube:
    """This rank's shard of a cube sharded over the default process group."""

    def __init__(self, extents, dtype, rank: int, world: int, block: int = 1, device: int = 0, group=None):
        self.extents = tuple(int(e) for e in extents)
        self.cube = Cube(self.extents, dtype, shard=(world, rank, block), device=device)
        self.dtype_code = self.cube.dtype_code
        self.rank, self.world, self.group = rank, world, group
        self._ws = None

    def _workspace(self, nq: int):
        import torch
        if self._ws is None or self._ws[0].numel() < nq:
            dev = torch.device("cuda", self.cube.device)
            self._ws = (torch.empty(nq, dtype=torch.int64, device=dev),
                        torch.empty(2 * nq, dtype=torch.int32, device=dev))
        return self._ws[0][:nq], self._ws[1][:2 * nq]

    def query_device(self, d_ranges, d_ops, d_results, stream=None):
        nq = d_ops.numel()
        psum, pext = self._workspace(nq)
        self.cube.partials_device(d_ranges, d_ops, psum, pext, nq=nq, stream=stream)
        if self.world > 1:
            exchange_partials(psum, pext, self.dtype_code, self.group)
        finalize_device(self.extents, self.dtype_code, nq, d_ranges, d_ops, psum, pext, d_results, stream=stream)

    def query(self, ranges, ops) -> np.ndarray:
        """Host arrays in, host results out (every rank gets every answer)."""
        import torch
        dev = torch.device("cuda", self.cube.device)
        rng = torch.from_numpy(np.ascontiguousarray(ranges, dtype=np.int64)).to(dev)
        opt = torch.from_numpy(np.ascontiguousarray(ops, dtype=np.int32)).to(dev)
        res = torch.empty(opt.numel() * RESULT_DTYPE.itemsize, dtype=torch.uint8, device=dev)
        self.query_device(rng, opt, res)
        return res.cpu().numpy().view(RESULT_DTYPE)
