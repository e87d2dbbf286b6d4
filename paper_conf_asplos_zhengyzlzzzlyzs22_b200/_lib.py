"""ctypes loader for lib/libastitch.so (the C ABI of include/astitch.h).

Argument marshalling only: no computation happens in Python.  If the shared
library is missing the import fails loudly -- there is no fallback path.
"""

from __future__ import annotations

import ctypes as ct
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("ASTITCH_LIB", os.path.join(_HERE, "lib", "libastitch.so"))

STATUS = {
    0: "ASTITCH_OK", 1: "ASTITCH_ERR_INVALID_ARGUMENT", 2: "ASTITCH_ERR_INVALID_GRAPH",
    3: "ASTITCH_ERR_UNSUPPORTED", 4: "ASTITCH_ERR_SHAPE", 5: "ASTITCH_ERR_RESOURCE",
    6: "ASTITCH_ERR_CUDA", 7: "ASTITCH_ERR_NCCL", 8: "ASTITCH_ERR_INTERNAL",
}

DTYPES = {"F32": 0, "BF16": 1, "F16": 2, "I32": 3}
KINDS = {"FULL": 0, "ROWVEC": 1, "COLVEC": 2, "SCALAR": 3, "LENGTHS": 4, "SEGMENTS": 5}
UNOPS = {n: i for i, n in enumerate(["NEG", "ABS", "EXP", "LOG", "TANH", "ERF", "SQRT", "RSQRT", "RCP",
                                     "SIGMOID", "GELU_TANH", "GELU_ERF", "GELU_TANH_GRAD"])}
BINOPS = {n: i for i, n in enumerate(["ADD", "SUB", "MUL", "DIV", "MAX", "MIN", "POW"])}
REDOPS = {"SUM": 0, "RMAX": 1}
AXES = {"ROW": 0, "COL": 1}

FLAG_NO_COMPILE = 1 << 0
FLAG_FORCE_GLOBAL = 1 << 1
FLAG_NO_PACK = 1 << 2
FLAG_NO_SPLIT = 1 << 3
FLAG_STRICT_SINGLE_KERNEL = 1 << 4
FLAG_NO_TMA = 1 << 5
FLAG_NO_PREFETCH = 1 << 6
FLAG_LAUNCH_CHECK = 1 << 7
FLAG_FORCE_SPLIT = 1 << 8
FLAG_NO_PDL = 1 << 9
FLAG_DEBUG_BARRIER = 1 << 10


class AstitchError(RuntimeError):
    def __init__(self, status: int, where: str, detail: str):
        self.status = status
        self.status_name = STATUS.get(status, str(status))
        super().__init__(f"{where}: {self.status_name}: {detail}")


class PlanDesc(ct.Structure):
    _fields_ = [("rows", ct.c_int64), ("cols", ct.c_int64), ("device", ct.c_int32),
                ("shard_rank", ct.c_int32), ("shard_world", ct.c_int32), ("flags", ct.c_uint32),
                ("sm_count", ct.c_int32), ("reserved", ct.c_int32)]


if not os.path.exists(LIB_PATH):
    raise ImportError(f"libastitch.so not found at {LIB_PATH}: run `python -m "
                      "paper_conf_asplos_zhengyzlzzzlyzs22_b200.build` (or __graft_entry__.build())")

lib = ct.CDLL(LIB_PATH)

_vp = ct.c_void_p
_i32p = ct.POINTER(ct.c_int32)
_sig = {
    "astitch_status_str": (ct.c_char_p, [ct.c_int]),
    "astitch_last_error": (ct.c_char_p, []),
    "astitch_abi_version": (ct.c_int, []),
    "astitch_graph_create": (ct.c_int, [ct.POINTER(_vp)]),
    "astitch_graph_destroy": (ct.c_int, [_vp]),
    "astitch_graph_input": (ct.c_int, [_vp, ct.c_int, ct.c_int, _i32p]),
    "astitch_graph_const": (ct.c_int, [_vp, ct.c_double, _i32p]),
    "astitch_graph_unary": (ct.c_int, [_vp, ct.c_int, ct.c_int32, _i32p]),
    "astitch_graph_binary": (ct.c_int, [_vp, ct.c_int, ct.c_int32, ct.c_int32, _i32p]),
    "astitch_graph_reduce": (ct.c_int, [_vp, ct.c_int, ct.c_int, ct.c_int32, _i32p]),
    "astitch_graph_broadcast": (ct.c_int, [_vp, ct.c_int, ct.c_int32, _i32p]),
    "astitch_graph_lengths": (ct.c_int, [_vp, ct.c_int64, _i32p]),
    "astitch_graph_set_mask": (ct.c_int, [_vp, ct.c_int32, ct.c_int64]),
    "astitch_graph_segments": (ct.c_int, [_vp, ct.c_int32, ct.c_int64, _i32p]),
    "astitch_segments_layout": (ct.c_int, [ct.c_int32, ct.POINTER(ct.c_int64), _i32p, _i32p,
                                           ct.POINTER(ct.c_int64), ct.POINTER(ct.c_int64)]),
    "astitch_graph_output": (ct.c_int, [_vp, ct.c_int32, ct.c_int, _i32p]),
    "astitch_plan": (ct.c_int, [_vp, ct.POINTER(PlanDesc), ct.POINTER(_vp)]),
    "astitch_plan_ex": (ct.c_int, [_vp, ct.POINTER(PlanDesc), ct.c_char_p, ct.POINTER(_vp)]),
    "astitch_set_cache_dir": (ct.c_int, [ct.c_char_p]),
    "astitch_plan_destroy": (ct.c_int, [_vp]),
    "astitch_plan_workspace_bytes": (ct.c_int, [_vp, ct.POINTER(ct.c_size_t)]),
    "astitch_plan_describe": (ct.c_int, [_vp, ct.c_char_p, ct.c_size_t, ct.POINTER(ct.c_size_t)]),
    "astitch_plan_source": (ct.c_int, [_vp, ct.c_int32, ct.c_char_p, ct.c_size_t, ct.POINTER(ct.c_size_t)]),
    "astitch_plan_cubin": (ct.c_int, [_vp, ct.c_int32, _vp, ct.c_size_t, ct.POINTER(ct.c_size_t)]),
    "astitch_plan_kernel_count": (ct.c_int, [_vp, _i32p]),
    "astitch_plan_io_count": (ct.c_int, [_vp, _i32p, _i32p]),
    "astitch_plan_io": (ct.c_int, [_vp, ct.c_int32, ct.c_int32, ct.POINTER(ct.c_int), ct.POINTER(ct.c_int)]),
    "astitch_workspace_init": (ct.c_int, [_vp, _vp, _vp]),
    "astitch_run": (ct.c_int, [_vp, ct.POINTER(_vp), ct.POINTER(_vp), _vp, _vp]),
    "astitch_run_sharded_host": (ct.c_int, [_vp, _vp, _vp, ct.POINTER(_vp), ct.POINTER(_vp), ct.POINTER(_vp),
                                             ct.POINTER(_vp), _vp, _vp]),
    "astitch_run_host": (ct.c_int, [_vp, ct.POINTER(_vp), ct.POINTER(_vp), ct.POINTER(_vp),
                                    ct.POINTER(_vp), _vp, _vp]),
    "astitch_run_host_pipelined": (ct.c_int, [_vp, ct.POINTER(_vp), ct.POINTER(_vp), ct.POINTER(_vp),
                                              ct.POINTER(_vp), _vp, _vp, ct.c_int32]),
    "astitch_comm_unique_id": (ct.c_int, [ct.c_char_p]),
    "astitch_comm_create": (ct.c_int, [ct.c_int32, ct.c_int32, ct.c_char_p, ct.c_int32, ct.POINTER(_vp)]),
    "astitch_comm_destroy": (ct.c_int, [_vp]),
    "astitch_run_sharded": (ct.c_int, [_vp, _vp, ct.POINTER(_vp), ct.POINTER(_vp), _vp, _vp]),
    "astitch_run_shard_stage": (ct.c_int, [_vp, ct.c_int32, ct.POINTER(_vp), ct.POINTER(_vp), _vp, _vp]),
    "astitch_plan_colpart": (ct.c_int, [_vp, ct.POINTER(ct.c_size_t), ct.POINTER(ct.c_size_t)]),
    "astitch_plan_colpart_ops": (ct.c_int, [_vp, _i32p, ct.c_size_t, ct.POINTER(ct.c_size_t)]),
    "astitch_peer_create": (ct.c_int, [_vp, ct.POINTER(_vp), ct.c_char_p]),
    "astitch_peer_open": (ct.c_int, [_vp, ct.c_int32, ct.c_char_p]),
    "astitch_peer_link": (ct.c_int, [_vp, ct.c_int32, _vp]),
    "astitch_peer_status": (ct.c_int, [_vp, _i32p]),
    "astitch_peer_destroy": (ct.c_int, [_vp]),
    "astitch_run_fused": (ct.c_int, [_vp, _vp, ct.POINTER(_vp), ct.POINTER(_vp), _vp, _vp]),
    "astitch_shard_rows": (ct.c_int, [ct.c_int64, ct.c_int32, ct.c_int32, ct.POINTER(ct.c_int64),
                                      ct.POINTER(ct.c_int64)]),
    "astitch_bench_barrier": (ct.c_int, [ct.c_int32, ct.c_int32, ct.c_int32, ct.c_int32, _vp, _vp]),
    "astitch_bench_copy": (ct.c_int, [ct.c_int32, _vp, _vp, ct.c_size_t, _vp]),
}
EXPORTED = tuple(_sig)

for _name, (_res, _args) in _sig.items():
    _f = getattr(lib, _name)
    _f.restype = _res
    _f.argtypes = _args


def check(status: int, where: str) -> None:
    if status != 0:
        detail = lib.astitch_last_error().decode(errors="replace")
        raise AstitchError(status, where, detail)


def ptr_array(ptrs) -> ct.Array:
    return (_vp * max(1, len(ptrs)))(*ptrs)
