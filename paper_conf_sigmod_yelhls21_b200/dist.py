"""Multi-GPU plumbing for the 1-D vertex-range partition.

One process per GPU.  Rank r owns rows [b_r, b_{r+1}) of the CSR (bounds from
``glp_partition``: equal vertex counts, or equal arc counts), keeps the owned
rows with GLOBAL column ids, and replicates the label array; the library
exchanges labels each iteration with an in-place NCCL all-gather.  This module
only slices the CSR and distributes the NCCL unique id through
``torch.distributed``; all per-iteration work happens inside libglp.so.
"""
from __future__ import annotations

import threading

import torch

from . import Graph, glp_local_group_create, glp_local_group_destroy, glp_nccl_unique_id, glp_partition


def shard_bounds(n: int, world: int, row_offsets=None, edge_balanced: bool = False):
    """Row bounds [b_0 = 0, ..., b_world = n] of every rank."""
    return glp_partition(n, world, row_offsets if edge_balanced else None, edge_balanced=edge_balanced)


def local_rows(row_offsets: torch.Tensor, col_idx: torch.Tensor, v_begin: int, v_end: int):
    """The owned rows of a global CSR: rebased offsets + their arcs (global ids)."""
    o0 = int(row_offsets[v_begin])
    o1 = int(row_offsets[v_end])
    off = (row_offsets[v_begin:v_end + 1] - o0).contiguous()
    col = col_idx[o0:o1].contiguous()
    return off, col


def broadcast_unique_id(group=None) -> bytes:
    """Rank 0 creates the 128-byte NCCL id; every rank receives it."""
    import torch.distributed as dist
    obj = [glp_nccl_unique_id() if dist.get_rank(group) == 0 else None]
    dist.broadcast_object_list(obj, src=0, group=group)
    return obj[0]


def distributed_graph(csr, group=None, edge_balanced: bool = False, stream=None) -> Graph:
    """Create this rank's share of `csr` (full graph on every rank) as a
    multi-GPU glp graph over the NCCL communicator of the process group."""
    import torch.distributed as dist
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    bounds = shard_bounds(csr.n, world, csr.row_offsets.cpu(), edge_balanced)
    vb, ve = bounds[rank], bounds[rank + 1]
    off, col = local_rows(csr.row_offsets, csr.col_idx, vb, ve)
    uid = broadcast_unique_id(group) if world > 1 else None
    dev = torch.cuda.current_device()
    return Graph(n=csr.n, row_offsets=off, col_idx=col, symmetric=csr.symmetric, rank=rank, nranks=world,
                 nccl_unique_id=uid,
                 v_begin=vb, v_end=ve, device=dev, stream=stream)


class LocalGroup:
    """P ranks of the 1-D partition in ONE process (glp_local_group): each rank
    is a Graph driven by its own host thread, and the library exchanges labels
    through the ranks' device buffers instead of NCCL.  With every rank on one
    GPU this runs libglp's real partitioned path (per-rank layout, pos/orig
    exchange, counter reduction, frontier-mark merge, sharded LLP histogram)
    where only one GPU is available.  Argument marshalling only."""

    def __init__(self, csr, nranks: int, edge_balanced: bool = False, bounds=None, device=None, weights=None):
        self.nranks = int(nranks)
        self.n = csr.n
        self.bounds = list(bounds) if bounds is not None else \
            shard_bounds(csr.n, self.nranks, csr.row_offsets.cpu(), edge_balanced)
        dev = torch.device("cuda", torch.cuda.current_device()) if device is None else torch.device(device)
        self.handle = glp_local_group_create(self.nranks)
        off = csr.row_offsets.to(dev)
        col = csr.col_idx.to(dev)
        self._parts = [local_rows(off, col, self.bounds[r], self.bounds[r + 1]) for r in range(self.nranks)]
        self._w = [None] * self.nranks
        if weights is not None:
            w = weights.to(dev).to(torch.int32)
            offc = off.cpu()
            self._w = [w[int(offc[self.bounds[r]]):int(offc[self.bounds[r + 1]])].contiguous()
                       for r in range(self.nranks)]
        torch.cuda.synchronize(dev)

        def make(r):
            o, c = self._parts[r]
            return Graph(n=csr.n, row_offsets=o, col_idx=c, symmetric=csr.symmetric, rank=r, nranks=self.nranks,
                         v_begin=self.bounds[r], v_end=self.bounds[r + 1], device=dev.index,
                         local_group=self.handle, weights=self._w[r])
        self.graphs = self._all(make)

    def _all(self, fn):
        """fn(rank) on every rank concurrently (the calls are collective)."""
        out = [None] * self.nranks
        err = [None] * self.nranks

        def body(r):
            try:
                out[r] = fn(r)
            except BaseException as e:  # re-raised below
                err[r] = e
        th = [threading.Thread(target=body, args=(r,)) for r in range(self.nranks)]
        for t in th:
            t.start()
        for t in th:
            t.join()
        for e in err:
            if e is not None:
                raise e
        return out

    def run(self, variant="classic", max_iters: int = 20, seeds=None, **kw):
        return self._all(lambda r: self.graphs[r].run(variant, max_iters, seeds, **kw))

    def labels(self, rank: int = 0, device="cpu"):
        return self.graphs[rank].labels(device)

    def iter_stats(self, rank: int = 0):
        return self.graphs[rank].iter_stats()

    def close(self):
        for g in getattr(self, "graphs", None) or []:
            if g is not None:
                g.close()
        self.graphs = []
        if getattr(self, "handle", None):
            glp_local_group_destroy(self.handle)
            self.handle = None

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()
