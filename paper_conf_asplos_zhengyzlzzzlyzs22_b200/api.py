"""Thin Python binding over the C ABI (include/astitch.h).

Names follow the C entry points; every call is argument marshalling (device
pointers and the caller's CUDA stream go straight to libastitch.so).  PyTorch
is used only to hold device memory and to name the current stream.
"""

from __future__ import annotations

import ctypes as ct
import json

from . import _lib
from ._lib import AstitchError, check, lib, ptr_array

_TORCH_DT = None


def _torch_dtype(dt: str):
    import torch
    return {"F32": torch.float32, "BF16": torch.bfloat16, "F16": torch.float16, "I32": torch.int32}[dt]


_DT_NAME = {v: k for k, v in _lib.DTYPES.items()}
_KIND_NAME = {v: k for k, v in _lib.KINDS.items()}


class Graph:
    """Op-graph IR builder (astitch_graph_*)."""

    def __init__(self):
        h = ct.c_void_p()
        check(lib.astitch_graph_create(ct.byref(h)), "astitch_graph_create")
        self._h = h
        self.names: dict[str, int] = {}
        self.ragged = None  # (nseg, elems) once astitch_graph_segments was called

    def __del__(self):
        h = getattr(self, "_h", None)
        if h is not None and h.value:
            lib.astitch_graph_destroy(h)
            self._h = None

    @property
    def handle(self):
        return self._h

    def _out(self):
        return ct.c_int32()

    def input(self, kind: str, dtype: str) -> int:
        v = self._out()
        check(lib.astitch_graph_input(self._h, _lib.KINDS[kind], _lib.DTYPES[dtype], ct.byref(v)),
              "astitch_graph_input")
        return v.value

    def lengths(self, rows_per_segment: int) -> int:
        v = self._out()
        check(lib.astitch_graph_lengths(self._h, int(rows_per_segment), ct.byref(v)), "astitch_graph_lengths")
        return v.value

    def set_mask(self, lengths: int, rows_per_segment: int) -> None:
        """astitch_graph_set_mask: bind an existing LENGTHS input (created with
        input("LENGTHS", "I32")) as the key-padding mask."""
        check(lib.astitch_graph_set_mask(self._h, int(lengths), int(rows_per_segment)), "astitch_graph_set_mask")

    def segments(self, nseg: int, elems: int) -> int:
        """Packed varlen rows (astitch_graph_segments): adds the int32 [nseg, 4]
        segment-table input; FULL tensors then hold `elems` packed elements."""
        v = self._out()
        check(lib.astitch_graph_segments(self._h, int(nseg), int(elems), ct.byref(v)), "astitch_graph_segments")
        self.ragged = (int(nseg), int(elems))
        return v.value

    def const(self, value: float) -> int:
        v = self._out()
        check(lib.astitch_graph_const(self._h, float(value), ct.byref(v)), "astitch_graph_const")
        return v.value

    def unary(self, op: str, a: int) -> int:
        v = self._out()
        check(lib.astitch_graph_unary(self._h, _lib.UNOPS[op], a, ct.byref(v)), "astitch_graph_unary")
        return v.value

    def binary(self, op: str, a: int, b: int) -> int:
        v = self._out()
        check(lib.astitch_graph_binary(self._h, _lib.BINOPS[op], a, b, ct.byref(v)), "astitch_graph_binary")
        return v.value

    def reduce(self, op: str, axis: str, a: int) -> int:
        v = self._out()
        check(lib.astitch_graph_reduce(self._h, _lib.REDOPS[op], _lib.AXES[axis], a, ct.byref(v)),
              "astitch_graph_reduce")
        return v.value

    def broadcast(self, axis: str, a: int) -> int:
        v = self._out()
        check(lib.astitch_graph_broadcast(self._h, _lib.AXES[axis], a, ct.byref(v)), "astitch_graph_broadcast")
        return v.value

    def output(self, v: int, dtype: str) -> int:
        idx = ct.c_int32()
        check(lib.astitch_graph_output(self._h, v, _lib.DTYPES[dtype], ct.byref(idx)), "astitch_graph_output")
        return idx.value

    @classmethod
    def from_spec(cls, spec: dict) -> "Graph":
        """Replay a declarative spec (workloads/specs.py format) through the builder."""
        g = cls()
        n = g.names
        mask = spec.get("mask")
        for name, kind, dtype in spec["inputs"]:
            if kind == "LENGTHS":
                assert mask is not None and mask["lengths"] == name
                n[name] = g.lengths(mask["rows_per_segment"])
            elif kind == "SEGMENTS":
                seg = spec["segments"]
                assert seg["table"] == name
                n[name] = g.segments(len(seg["seg_rows"]), seg["elems"])
            else:
                n[name] = g.input(kind, dtype)
        for op in spec["ops"]:
            name, typ = op[0], op[1]
            if typ == "const":
                n[name] = g.const(op[2])
            elif typ == "unary":
                n[name] = g.unary(op[2], n[op[3]])
            elif typ == "binary":
                n[name] = g.binary(op[2], n[op[3]], n[op[4]])
            elif typ == "reduce":
                n[name] = g.reduce(op[2], op[3], n[op[4]])
            elif typ == "broadcast":
                n[name] = g.broadcast(op[2], n[op[3]])
            else:
                raise ValueError(typ)
        for name, dtype in spec["outputs"]:
            g.output(n[name], dtype)
        return g


def _stream_ptr(stream):
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


class Plan:
    """A planned + JIT-compiled stitch op (astitch_plan)."""

    def __init__(self, graph: Graph, rows: int, cols: int, device: int = 0, flags: int = 0,
                 shard_rank: int = 0, shard_world: int = 1, sm_count: int = 0, tune: str | dict | None = None):
        """`tune`: explicit planner overrides for experiments / tests
        (astitch_plan_ex), "key=value,..." or a dict, e.g. {"threads": 256}."""
        d = _lib.PlanDesc(rows=int(rows), cols=int(cols), device=int(device), shard_rank=int(shard_rank),
                          shard_world=int(shard_world), flags=int(flags), sm_count=int(sm_count), reserved=0)
        h = ct.c_void_p()
        if isinstance(tune, dict):
            tune = ",".join(f"{k}={int(v)}" for k, v in tune.items())
        if tune:
            check(lib.astitch_plan_ex(graph.handle, ct.byref(d), tune.encode(), ct.byref(h)), "astitch_plan_ex")
        else:
            check(lib.astitch_plan(graph.handle, ct.byref(d), ct.byref(h)), "astitch_plan")
        self._h = h
        self.rows, self.cols, self.device = int(rows), int(cols), int(device)
        self.ragged = graph.ragged
        ni, no = ct.c_int32(), ct.c_int32()
        check(lib.astitch_plan_io_count(h, ct.byref(ni), ct.byref(no)), "astitch_plan_io_count")
        self.inputs = [self._io(0, i) for i in range(ni.value)]
        self.outputs = [self._io(1, i) for i in range(no.value)]
        self._ws_cache = None   # workspace per stream (concurrent runs need distinct workspaces)
        self._ws_by_stream = {}

    def __del__(self):
        h = getattr(self, "_h", None)
        if h is not None and h.value:
            lib.astitch_plan_destroy(h)
            self._h = None

    def _io(self, is_out, i):
        k, d = ct.c_int(), ct.c_int()
        check(lib.astitch_plan_io(self._h, is_out, i, ct.byref(k), ct.byref(d)), "astitch_plan_io")
        return (_KIND_NAME[k.value], _DT_NAME[d.value])

    @property
    def handle(self):
        return self._h

    def describe(self) -> dict:
        n = ct.c_size_t()
        check(lib.astitch_plan_describe(self._h, None, 0, ct.byref(n)), "astitch_plan_describe")
        buf = ct.create_string_buffer(n.value + 1)
        check(lib.astitch_plan_describe(self._h, buf, n.value + 1, ct.byref(n)), "astitch_plan_describe")
        return json.loads(buf.value.decode())

    def kernel_count(self) -> int:
        n = ct.c_int32()
        check(lib.astitch_plan_kernel_count(self._h, ct.byref(n)), "astitch_plan_kernel_count")
        return n.value

    def source(self, k: int = 0) -> str:
        n = ct.c_size_t()
        check(lib.astitch_plan_source(self._h, k, None, 0, ct.byref(n)), "astitch_plan_source")
        buf = ct.create_string_buffer(n.value + 1)
        check(lib.astitch_plan_source(self._h, k, buf, n.value + 1, ct.byref(n)), "astitch_plan_source")
        return buf.value.decode()

    def cubin(self, k: int = 0) -> bytes:
        n = ct.c_size_t()
        check(lib.astitch_plan_cubin(self._h, k, None, 0, ct.byref(n)), "astitch_plan_cubin")
        buf = ct.create_string_buffer(max(1, n.value))
        check(lib.astitch_plan_cubin(self._h, k, buf, n.value, ct.byref(n)), "astitch_plan_cubin")
        return buf.raw[: n.value]

    def workspace_bytes(self) -> int:
        n = ct.c_size_t()
        check(lib.astitch_plan_workspace_bytes(self._h, ct.byref(n)), "astitch_plan_workspace_bytes")
        return n.value

    # -------------------------------------------------------------- torch helpers
    def io_shape(self, kind: str, rows: int | None = None, nseg: int | None = None):
        R = self.rows if rows is None else rows
        if kind == "FULL":
            return (self.ragged[1],) if self.ragged else (R, self.cols)
        if kind == "SEGMENTS":
            return (self.ragged[0], 4)
        if kind == "ROWVEC":
            return (R,)
        if kind == "COLVEC":
            return (self.cols,)
        if kind == "LENGTHS":
            return (nseg,)
        raise ValueError(kind)

    def alloc_outputs(self, device=None):
        import torch
        dev = torch.device("cuda", self.device) if device is None else device
        return [torch.empty(self.io_shape(k), dtype=_torch_dtype(d), device=dev) for k, d in self.outputs]

    def alloc_workspace(self, stream=None):
        """Allocate (as a torch uint8 tensor) and initialise a workspace once."""
        import torch
        n = self.workspace_bytes()
        if n == 0:
            return None
        ws = torch.empty(n + 256, dtype=torch.uint8, device=torch.device("cuda", self.device))
        off = (-ws.data_ptr()) % 256
        ws = ws[off: off + n]
        check(lib.astitch_workspace_init(self._h, ct.c_void_p(ws.data_ptr()), ct.c_void_p(_stream_ptr(stream))),
              "astitch_workspace_init")
        return ws

    def _numel(self, kind: str):
        if kind == "LENGTHS":
            return None  # one length per segment of rows_per_segment rows (checked by the caller's spec)
        n = 1
        for d in self.io_shape(kind):
            n *= d
        return n

    def check_io(self, inputs, outputs, device: bool = True) -> None:
        """Validate tensors against the plan's I/O list (count, dtype, element
        count, contiguity, CUDA placement): the C ABI sees only base pointers,
        so a strided view or a wrong dtype would otherwise be read silently."""
        for what, ts, decl in (("input", inputs, self.inputs), ("output", outputs, self.outputs)):
            if len(ts) != len(decl):
                raise ValueError(f"expected {len(decl)} {what}s, got {len(ts)}")
            for i, (t, (kind, dt)) in enumerate(zip(ts, decl)):
                want = _torch_dtype(dt)
                if t.dtype != want:
                    raise ValueError(f"{what} {i} ({kind}): dtype {t.dtype}, plan expects {want}")
                if not t.is_contiguous():
                    raise ValueError(f"{what} {i} ({kind}): tensor is not contiguous")
                n = self._numel(kind)
                if n is not None and t.numel() != n:
                    raise ValueError(f"{what} {i} ({kind}): {t.numel()} elements, plan expects {n}")
                if device and not t.is_cuda:
                    raise ValueError(f"{what} {i} ({kind}): expected a CUDA tensor")
                if device and t.device.index is not None and t.device.index != self.device:
                    raise ValueError(f"{what} {i} ({kind}): tensor on cuda:{t.device.index}, plan is for cuda:{self.device}")

    def _stream_ws(self, stream):
        """The plan's cached workspace for `stream` (one per stream: the grid
        barrier words of a workspace must not be shared by concurrent runs)."""
        if self.workspace_bytes() == 0:
            return None
        sp = _stream_ptr(stream)
        ws = self._ws_by_stream.get(sp)
        if ws is None:
            ws = self._ws_by_stream[sp] = self.alloc_workspace(stream)
            if self._ws_cache is None:
                self._ws_cache = ws
        return ws

    def _check_stream(self, stream):
        if stream is not None and not isinstance(stream, int):
            dev = getattr(stream, "device", None)
            if dev is not None and getattr(dev, "index", None) is not None and dev.index != self.device:
                raise ValueError(f"stream is on cuda:{dev.index}, plan is for cuda:{self.device}")

    def run(self, inputs, outputs, ws=None, stream=None) -> None:
        """astitch_run on device tensors (in declaration order) on `stream`."""
        self.check_io(inputs, outputs)
        self._check_stream(stream)
        if ws is None:
            ws = self._stream_ws(stream)
        ins = ptr_array([t.data_ptr() for t in inputs])
        outs = ptr_array([t.data_ptr() for t in outputs])
        check(lib.astitch_run(self._h, ins, outs, ct.c_void_p(ws.data_ptr() if ws is not None else 0),
                              ct.c_void_p(_stream_ptr(stream))), "astitch_run")

    def bind(self, inputs, outputs, ws=None, stream=None):
        """Pre-marshalled astitch_run for repeated eager calls on the same
        buffers and stream: returns a no-argument callable whose only work per
        call is the C-ABI call (pointer arrays, workspace and stream are
        resolved once here; the tensors are kept alive by the callable)."""
        self.check_io(inputs, outputs)
        self._check_stream(stream)
        if ws is None:
            ws = self._stream_ws(stream)
        ins = ptr_array([t.data_ptr() for t in inputs])
        outs = ptr_array([t.data_ptr() for t in outputs])
        w = ct.c_void_p(ws.data_ptr() if ws is not None else 0)
        s = ct.c_void_p(_stream_ptr(stream))
        fn, h = lib.astitch_run, self._h
        keep = (self, list(inputs), list(outputs), ws)

        def run() -> None:
            st = fn(h, ins, outs, w, s)
            if st:
                check(st, "astitch_run")

        run.keep = keep
        return run

    def run_host(self, host_inputs, host_outputs, dev_inputs, dev_outputs, ws=None, stream=None,
                 chunks: int = 1) -> None:
        """astitch_run_host (chunks == 1) / astitch_run_host_pipelined (chunks > 1):
        H2D inputs, stitched kernel(s), D2H outputs, asynchronous on `stream`."""
        self.check_io(host_inputs, host_outputs, device=False)
        self.check_io(dev_inputs, dev_outputs)
        self._check_stream(stream)
        if ws is None:
            ws = self._stream_ws(stream)
        hi = ptr_array([t.data_ptr() for t in host_inputs])
        ho = ptr_array([t.data_ptr() for t in host_outputs])
        di = ptr_array([t.data_ptr() for t in dev_inputs])
        do = ptr_array([t.data_ptr() for t in dev_outputs])
        w = ct.c_void_p(ws.data_ptr() if ws is not None else 0)
        s = ct.c_void_p(_stream_ptr(stream))
        if chunks > 1:
            check(lib.astitch_run_host_pipelined(self._h, hi, ho, di, do, w, s, int(chunks)),
                  "astitch_run_host_pipelined")
        else:
            check(lib.astitch_run_host(self._h, hi, ho, di, do, w, s), "astitch_run_host")


def plan(graph: Graph, rows: int, cols: int, device: int = 0, flags: int = 0, **kw) -> Plan:
    return Plan(graph, rows, cols, device=device, flags=flags, **kw)


def segments_layout(seg_rows, seg_cols):
    """astitch_segments_layout: canonical packed varlen table for segments of
    seg_rows[s] x seg_cols[s] (pitch = cols rounded up to 8 elements).
    Returns (table int32 [nseg, 4] as a list of rows, total rows, total elements)."""
    nseg = len(seg_rows)
    assert len(seg_cols) == nseg
    r = (ct.c_int64 * nseg)(*[int(x) for x in seg_rows])
    c = (ct.c_int32 * nseg)(*[int(x) for x in seg_cols])
    t = (ct.c_int32 * (4 * nseg))()
    rows, elems = ct.c_int64(), ct.c_int64()
    check(lib.astitch_segments_layout(nseg, r, c, t, ct.byref(rows), ct.byref(elems)), "astitch_segments_layout")
    return [list(t[4 * s: 4 * s + 4]) for s in range(nseg)], rows.value, elems.value


def set_cache_dir(path: str | None) -> None:
    """astitch_set_cache_dir: on-disk cubin cache directory (None / "" = off)."""
    check(lib.astitch_set_cache_dir(path.encode() if path else None), "astitch_set_cache_dir")


def shard_rows(rows: int, world: int, rank: int) -> tuple[int, int]:
    b, c = ct.c_int64(), ct.c_int64()
    check(lib.astitch_shard_rows(int(rows), int(world), int(rank), ct.byref(b), ct.byref(c)), "astitch_shard_rows")
    return b.value, c.value


def bench_barrier(device: int, blocks: int, threads: int, iters: int, ws, stream=None) -> None:
    check(lib.astitch_bench_barrier(device, blocks, threads, iters, ct.c_void_p(ws.data_ptr()),
                                    ct.c_void_p(_stream_ptr(stream))), "astitch_bench_barrier")


def bench_copy(device: int, src, dst, nbytes: int, stream=None) -> None:
    check(lib.astitch_bench_copy(device, ct.c_void_p(src.data_ptr()), ct.c_void_p(dst.data_ptr()), int(nbytes),
                                 ct.c_void_p(_stream_ptr(stream))), "astitch_bench_copy")


__all__ = ["Graph", "Plan", "plan", "segments_layout", "shard_rows", "set_cache_dir", "bench_barrier", "bench_copy", "AstitchError"]
