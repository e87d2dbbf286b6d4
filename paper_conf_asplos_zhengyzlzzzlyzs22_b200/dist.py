"""Row-sharded multi-GPU execution (BASELINE north_star (4)).

One process per GPU.  torch.distributed is the plumbing only: it bootstraps
the NCCL communicator of libastitch (the ncclUniqueId is broadcast through the
process group) and provides barriers for timing.  The data path is entirely in
libastitch: astitch_run_sharded launches the stitched kernel on the rank's row
slice and, when the subgraph has a column reduction, ONE ncclAllReduce of the
fp32 column partials followed by the column-consumer epilogue kernel.
"""

from __future__ import annotations

import ctypes as ct

from . import _lib
from ._lib import check, lib, ptr_array
from .api import Graph, Plan, _stream_ptr, shard_rows


class Comm:
    """NCCL communicator owned by libastitch (astitch_comm_*)."""

    def __init__(self, world: int, rank: int, device: int, unique_id: bytes):
        assert len(unique_id) == 128
        h = ct.c_void_p()
        check(lib.astitch_comm_create(world, rank, unique_id, device, ct.byref(h)), "astitch_comm_create")
        self._h = h
        self.world, self.rank, self.device = world, rank, device

    @staticmethod
    def unique_id() -> bytes:
        buf = ct.create_string_buffer(128)
        check(lib.astitch_comm_unique_id(buf), "astitch_comm_unique_id")
        return buf.raw

    @classmethod
    def from_process_group(cls, device: int, group=None) -> "Comm":
        import torch.distributed as dist
        rank, world = dist.get_rank(group), dist.get_world_size(group)
        obj = [cls.unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0, group=group)
        return cls(world, rank, device, obj[0])

    def __del__(self):
        h = getattr(self, "_h", None)
        if h is not None and h.value:
            lib.astitch_comm_destroy(h)
            self._h = None

    @property
    def handle(self):
        return self._h


class ShardedPlan:
    """The rank's plan over its contiguous row slice of an [R, C] problem."""

    def __init__(self, graph: Graph, rows: int, cols: int, world: int, rank: int, device: int,
                 comm: Comm | None = None, flags: int = 0):
        self.row_begin, self.row_count = shard_rows(rows, world, rank)
        self.plan = Plan(graph, self.row_count, cols, device=device, flags=flags, shard_rank=rank,
                         shard_world=world)
        self.comm = comm
        self.world, self.rank = world, rank

    def run(self, inputs, outputs, ws=None, stream=None) -> None:
        p = self.plan
        if ws is None and p.workspace_bytes() > 0:
            if p._ws_cache is None:
                p._ws_cache = p.alloc_workspace(stream)
            ws = p._ws_cache
        ins = ptr_array([t.data_ptr() for t in inputs])
        outs = ptr_array([t.data_ptr() for t in outputs])
        check(lib.astitch_run_sharded(p.handle, self.comm.handle if self.comm else None, ins, outs,
                                      ct.c_void_p(ws.data_ptr() if ws is not None else 0),
                                      ct.c_void_p(_stream_ptr(stream))), "astitch_run_sharded")

    def run_stage(self, stage: int, inputs, outputs, ws, stream=None) -> None:
        """astitch_run_shard_stage: 0 = stitched kernel leaving rank-local column
        totals in ws; 1 = column consumers reading the combined totals."""
        ins = ptr_array([t.data_ptr() for t in inputs])
        outs = ptr_array([t.data_ptr() for t in outputs])
        check(lib.astitch_run_shard_stage(self.plan.handle, int(stage), ins, outs,
                                          ct.c_void_p(ws.data_ptr() if ws is not None else 0),
                                          ct.c_void_p(_stream_ptr(stream))), "astitch_run_shard_stage")

    def colpart(self):
        """(byte offset in the workspace, float count) of the column totals."""
        off, n = ct.c_size_t(), ct.c_size_t()
        check(lib.astitch_plan_colpart(self.plan.handle, ct.byref(off), ct.byref(n)), "astitch_plan_colpart")
        return off.value, n.value

    def kernels_per_run(self) -> int:
        d = self.plan.describe()
        if self.world > 1 and d["shard_kernels"] > 0:
            return d["shard_kernels"]
        return d["kernel_count"]


def partition_by_weight(weights, world: int):
    """Contiguous partition of units (e.g. C3's 64 batches, weighted by their
    bytes) into `world` ranges with balanced total weight.  Pure host logic."""
    n = len(weights)
    total = float(sum(weights))
    bounds, acc, k = [0], 0.0, 1
    for i, w in enumerate(weights):
        acc += w
        while k < world and acc >= total * k / world and len(bounds) < world:
            bounds.append(i + 1)
            k += 1
    while len(bounds) < world:
        bounds.append(n)
    bounds.append(n)
    return [(bounds[r], bounds[r + 1]) for r in range(world)]


__all__ = ["Comm", "ShardedPlan", "partition_by_weight", "_lib"]
