"""Row-sharded multi-GPU execution (BASELINE north_star (4)).

One process per GPU.  torch.distributed is the plumbing only: it bootstraps
the NCCL communicator of libastitch (the ncclUniqueId is broadcast through the
process group) and provides barriers for timing.  The data path is entirely in
libastitch.  When the subgraph has a column reduction, the rank-local fp32
column totals are combined either INSIDE the stitched kernel over peer memory
(PeerExchange + astitch_run_fused: one kernel per rank, NVLink P2P stores and
flags) or by ONE ncclAllReduce between the stitched kernel and the
column-consumer epilogue (Comm + astitch_run_sharded).
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


class PeerExchange:
    """Exchange buffer of the fused sharded run (astitch_peer_*): this rank's
    buffer plus the mapping of every other rank's (CUDA IPC handles between
    processes, or direct links between ranks living in one process)."""

    def __init__(self, plan: Plan):
        h = ct.c_void_p()
        buf = ct.create_string_buffer(64)
        check(lib.astitch_peer_create(plan.handle, ct.byref(h), buf), "astitch_peer_create")
        self._h = h
        self.ipc_handle = buf.raw

    def open(self, rank: int, ipc_handle: bytes) -> None:
        check(lib.astitch_peer_open(self._h, int(rank), ipc_handle), "astitch_peer_open")

    def link(self, rank: int, other: "PeerExchange") -> None:
        check(lib.astitch_peer_link(self._h, int(rank), other._h), "astitch_peer_link")

    def timed_out(self) -> bool:
        v = ct.c_int32()
        check(lib.astitch_peer_status(self._h, ct.byref(v)), "astitch_peer_status")
        return bool(v.value)

    @classmethod
    def from_process_group(cls, plan: Plan, group=None) -> "PeerExchange":
        """One process per GPU: all-gather the IPC handles and map every peer."""
        import torch.distributed as dist
        x = cls(plan)
        handles = [None] * dist.get_world_size(group)
        dist.all_gather_object(handles, x.ipc_handle, group=group)
        me = dist.get_rank(group)
        for r, hnd in enumerate(handles):
            if r != me:
                x.open(r, hnd)
        return x

    def __del__(self):
        h = getattr(self, "_h", None)
        if h is not None and h.value and lib is not None:
            lib.astitch_peer_destroy(h)
            self._h = None

    @property
    def handle(self):
        return self._h


class ShardedPlan:
    """The rank's plan over its contiguous row slice of an [R, C] problem.

    A column reduction over the shards is combined either inside the stitched
    kernel over peer memory (`peer`: astitch_run_fused, one kernel) or with an
    NCCL allreduce between the stitched kernel and an epilogue (`comm`:
    astitch_run_sharded)."""

    def __init__(self, graph: Graph, rows: int, cols: int, world: int, rank: int, device: int,
                 comm: Comm | None = None, flags: int = 0, sm_count: int = 0, tune=None, row_range=None):
        """row_range: (row_begin, row_count) of this rank when the rows are not
        split evenly (e.g. masked batches balanced by bytes, `mask_row_ranges`);
        default: astitch_shard_rows' contiguous even split."""
        if row_range is None:
            self.row_begin, self.row_count = shard_rows(rows, world, rank)
        else:
            self.row_begin, self.row_count = int(row_range[0]), int(row_range[1])
        self.plan = Plan(graph, self.row_count, cols, device=device, flags=flags, shard_rank=rank,
                         shard_world=world, sm_count=sm_count, tune=tune)
        self.comm = comm
        self.peer: PeerExchange | None = None
        self.world, self.rank = world, rank

    def needs_exchange(self) -> bool:
        return self.world > 1 and self.plan.describe()["shard_kernels"] > 0

    def _ws(self, ws, stream):
        return self.plan._stream_ws(stream) if ws is None else ws

    def run(self, inputs, outputs, ws=None, stream=None) -> None:
        p = self.plan
        p.check_io(inputs, outputs)
        ws = self._ws(ws, stream)
        ins = ptr_array([t.data_ptr() for t in inputs])
        outs = ptr_array([t.data_ptr() for t in outputs])
        w = ct.c_void_p(ws.data_ptr() if ws is not None else 0)
        s = ct.c_void_p(_stream_ptr(stream))
        if self.peer is not None:
            check(lib.astitch_run_fused(p.handle, self.peer.handle, ins, outs, w, s), "astitch_run_fused")
            return
        check(lib.astitch_run_sharded(p.handle, self.comm.handle if self.comm else None, ins, outs, w, s),
              "astitch_run_sharded")

    def run_host(self, host_inputs, host_outputs, dev_inputs, dev_outputs, ws=None, stream=None) -> None:
        """astitch_run_sharded_host: H2D of this rank's inputs, the sharded
        (fused or NCCL) run, D2H of its outputs, asynchronous on `stream`."""
        p = self.plan
        p.check_io(host_inputs, host_outputs, device=False)
        p.check_io(dev_inputs, dev_outputs)
        ws = self._ws(ws, stream)
        arr = lambda ts: ptr_array([t.data_ptr() for t in ts])  # noqa: E731
        check(lib.astitch_run_sharded_host(p.handle, self.comm.handle if self.comm else None,
                                           self.peer.handle if self.peer is not None else None,
                                           arr(host_inputs), arr(host_outputs), arr(dev_inputs), arr(dev_outputs),
                                           ct.c_void_p(ws.data_ptr() if ws is not None else 0),
                                           ct.c_void_p(_stream_ptr(stream))), "astitch_run_sharded_host")

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

    def colpart_ops(self):
        """Per colpart slot: "sum" (fp32 totals, combine by fp32 sum) or "max"
        (int32 order keys, combine by int32 max); astitch_plan_colpart_ops."""
        n = ct.c_size_t()
        buf = (ct.c_int32 * 64)()
        check(lib.astitch_plan_colpart_ops(self.plan.handle, buf, 64, ct.byref(n)), "astitch_plan_colpart_ops")
        return ["max" if buf[i] == 1 else "sum" for i in range(n.value)]

    def kernels_per_run(self) -> int:
        d = self.plan.describe()
        if self.world > 1 and d["shard_kernels"] > 0 and self.peer is None:
            return d["shard_kernels"]
        return d["kernel_count"]


def partition_by_weight(weights, world: int):
    """Contiguous partition of units (e.g. C3's 64 batches, weighted by their
    bytes) into `world` ranges minimising the largest range weight (the
    slowest rank): binary search on that bound, each probe a greedy left-to-
    right fill.  Pure host logic; returns [(begin, end)] per rank."""
    w = [float(x) for x in weights]
    n = len(w)
    if n == 0:
        return [(0, 0)] * world

    def fill(cap):
        bounds, acc = [0], 0.0
        for i, x in enumerate(w):
            if acc + x > cap and acc > 0:
                bounds.append(i)
                acc = 0.0
            acc += x
        return bounds

    lo, hi = max(w), sum(w)
    for _ in range(100):
        mid = (lo + hi) / 2
        if len(fill(mid)) <= world:
            hi = mid
        else:
            lo = mid
    bounds = fill(hi)
    while len(bounds) < world:
        bounds.append(n)
    bounds.append(n)
    return [(bounds[r], bounds[r + 1]) for r in range(world)]


def mask_row_ranges(lengths, rows_per_segment: int, cols: int, rows: int, world: int,
                    in_bytes: int = 2, out_bytes: int = 2):
    """Row shards of a key-padding-masked problem: whole
    mask segments (batches) per rank, contiguous, balanced by each segment's
    compulsory bytes rows_per_segment x (in_bytes x L_b + out_bytes x cols)
    (valid-prefix reads + full-row writes).  Returns [(row_begin, row_count)]."""
    nseg = -(-rows // rows_per_segment)
    w = []
    for s_ in range(nseg):
        nr = min(rows_per_segment, rows - s_ * rows_per_segment)
        L = min(max(int(lengths[s_]), 0), cols)
        w.append(nr * (in_bytes * L + out_bytes * cols))
    out = []
    for a, b in partition_by_weight(w, world):
        r0 = a * rows_per_segment
        r1 = min(rows, b * rows_per_segment)
        out.append((r0, max(0, r1 - r0)))
    return out


__all__ = ["Comm", "PeerExchange", "ShardedPlan", "partition_by_weight", "mask_row_ranges", "_lib"]
