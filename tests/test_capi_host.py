"""Host-only tests of the C-ABI library: it loads without a GPU, exports every
symbol include/astitch.h declares, and returns the documented status codes."""

import ctypes as ct
import json
import os
import re

import pytest

import paper_conf_asplos_zhengyzlzzzlyzs22_b200 as A
from paper_conf_asplos_zhengyzlzzzlyzs22_b200 import _lib
from workloads import specs

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_symbols():
    text = open(os.path.join(ROOT, "include", "astitch.h")).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(astitch_[a-z_]+)\s*\(", text)))


def test_library_exports_every_header_symbol():
    syms = header_symbols()
    assert len(syms) >= 30
    for s in syms:
        assert hasattr(_lib.lib, s), f"libastitch.so does not export {s}"
    assert set(syms) == set(_lib.EXPORTED)
    assert _lib.lib.astitch_abi_version() == 1


def test_library_has_no_cuda_link_dependency():
    # libcuda / libnvrtc / libnccl are dlopen'ed lazily: loading works without a GPU
    out = os.popen(f"ldd {_lib.LIB_PATH}").read()
    for bad in ("libcuda.so", "libnvrtc", "libnccl", "libcudart"):
        assert bad not in out, out


def test_status_strings():
    for code, name in _lib.STATUS.items():
        assert _lib.lib.astitch_status_str(code).decode() == name


def _st(fn, *args):
    return fn(*args)


def test_builder_errors():
    g = A.Graph()
    x = g.input("FULL", "F32")
    r = g.input("ROWVEC", "F32")
    with pytest.raises(A.AstitchError) as e:
        g.binary("ADD", x, r)                     # kind mismatch -> INVALID_GRAPH
    assert e.value.status == 2
    with pytest.raises(A.AstitchError) as e:
        g.reduce("SUM", "ROW", r)                 # reduce of a ROWVEC -> UNSUPPORTED
    assert e.value.status == 3
    with pytest.raises(A.AstitchError) as e:
        g.broadcast("COL", r)                     # broadcast COL needs COLVEC -> INVALID_GRAPH
    assert e.value.status == 2
    v = ct.c_int32()
    assert _lib.lib.astitch_graph_unary(g.handle, 99, x, ct.byref(v)) == 1      # bad enum
    assert _lib.lib.astitch_graph_unary(g.handle, 0, 12345, ct.byref(v)) == 1   # bad operand
    assert _lib.lib.astitch_graph_unary(g.handle, 0, x, None) == 1              # NULL out
    assert _lib.lib.astitch_graph_input(g.handle, 3, 0, ct.byref(v)) == 1       # SCALAR input
    L = g.lengths(8)
    with pytest.raises(A.AstitchError):
        g.lengths(8)                              # one mask per graph
    with pytest.raises(A.AstitchError):
        g.unary("EXP", L)                         # LENGTHS is not an operand


def _plan_status(spec, rows, cols, flags=_lib.FLAG_NO_COMPILE):
    g = A.Graph.from_spec(spec)
    d = _lib.PlanDesc(rows=rows, cols=cols, device=-1, shard_rank=0, shard_world=1, flags=flags)
    h = ct.c_void_p()
    s = _lib.lib.astitch_plan(g.handle, ct.byref(d), ct.byref(h))
    if s == 0:
        _lib.lib.astitch_plan_destroy(h)
    return s


def test_plan_shape_errors():
    spec = specs.get("C1")
    assert _plan_status(spec, 32, 0) == 4          # cols < 1
    assert _plan_status(spec, -1, 128) == 4        # rows < 0
    assert _plan_status(spec, 1 << 41, 1 << 30) == 4
    assert _plan_status(spec, 0, 128) == 0         # rows = 0 is a valid (no-op) plan
    g = A.Graph()
    g.input("FULL", "F32")
    d = _lib.PlanDesc(rows=4, cols=4, device=-1, shard_world=1, flags=_lib.FLAG_NO_COMPILE)
    h = ct.c_void_p()
    assert _lib.lib.astitch_plan(g.handle, ct.byref(d), ct.byref(h)) == 2        # no outputs


def test_run_on_host_only_plan_fails_loudly():
    spec = specs.get("C1")
    p = A.Plan(A.Graph.from_spec(spec), 32, 128, device=-1, flags=A.FLAG_NO_COMPILE)
    ins = _lib.ptr_array([16])
    outs = _lib.ptr_array([32])
    s = _lib.lib.astitch_run(p.handle, ins, outs, None, None)
    assert s == 1
    assert "without a device" in _lib.lib.astitch_last_error().decode()
    # misaligned pointer
    s = _lib.lib.astitch_run(p.handle, _lib.ptr_array([17]), outs, None, None)
    assert s == 1 and "aligned" in _lib.lib.astitch_last_error().decode()


def test_shard_rows_partition():
    for R in (0, 1, 7, 1_048_576, 524_289):
        for g in (1, 2, 3, 4, 8):
            total, nxt = 0, 0
            for r in range(g):
                b, c = A.shard_rows(R, g, r)
                assert b == nxt and c in (R // g, R // g + 1)
                nxt, total = b + c, total + c
            assert total == R
    with pytest.raises(A.AstitchError):
        A.shard_rows(10, 2, 2)


def test_colpart_ops_per_slot():
    """astitch_plan_colpart_ops: the combine each colpart slot needs (SUM
    totals vs RMAX order keys), in colpart slot order; a too-small buffer is
    an error that still reports the count."""
    from paper_conf_asplos_zhengyzlzzzlyzs22_b200.dist import ShardedPlan
    spec = {"name": "mix", "rows": 1000, "cols": 64, "inputs": [("x", "FULL", "F32")], "mask": None,
            "ops": [("s", "reduce", "SUM", "COL", "x"), ("m", "reduce", "RMAX", "COL", "x")],
            "outputs": [("s", "F32"), ("m", "F32")]}
    sp = ShardedPlan(A.Graph.from_spec(spec), 1000, 64, 2, 1, -1, flags=A.FLAG_NO_COMPILE)
    assert sorted(sp.colpart_ops()) == ["max", "sum"]
    assert sp.colpart()[1] == 2 * 64
    n = ct.c_size_t()
    buf = (ct.c_int32 * 1)()
    assert _lib.lib.astitch_plan_colpart_ops(sp.plan.handle, buf, 1, ct.byref(n)) != 0 and n.value == 2
    row = specs.get("C2", rows=64)
    sp2 = ShardedPlan(A.Graph.from_spec(row), 64, 768, 2, 0, -1, flags=A.FLAG_NO_COMPILE)
    assert sp2.colpart_ops() == [] and _lib.lib.astitch_plan_colpart_ops(sp2.plan.handle, None, 0, ct.byref(n)) == 0


def test_io_signature_and_workspace():
    spec = specs.get("C5", rows=4096)
    p = A.Plan(A.Graph.from_spec(spec), 4096, 1024, device=-1, flags=A.FLAG_NO_COMPILE)
    assert p.inputs == [("FULL", "BF16"), ("FULL", "BF16"), ("COLVEC", "F32")]
    assert p.outputs == [("FULL", "BF16"), ("COLVEC", "F32"), ("COLVEC", "F32")]
    assert p.workspace_bytes() > 0
    spec = specs.get("C3", rows=8192)
    p = A.Plan(A.Graph.from_spec(spec), 8192, 512, device=-1, flags=A.FLAG_NO_COMPILE)
    assert p.inputs == [("FULL", "BF16"), ("LENGTHS", "I32")]
    assert p.workspace_bytes() == 256                       # tma_team: tile counter + done counter
    spec = specs.get("C2", rows=4096)
    p = A.Plan(A.Graph.from_spec(spec), 4096, 768, device=-1, flags=A.FLAG_NO_COMPILE)
    assert p.workspace_bytes() == 0                         # register row teams need none


def test_binding_checks_tensors_against_the_plan():
    """The binding validates count, dtype, element count and contiguity before
    a pointer crosses the C ABI (host tensors here; device placement on GPU)."""
    import torch
    from workloads import specs
    spec = specs.get("C5", rows=64, cols=32)
    p = A.Plan(A.Graph.from_spec(spec), 64, 32, device=-1, flags=A.FLAG_NO_COMPILE)
    ins = [torch.zeros(64, 32, dtype=torch.bfloat16), torch.zeros(64, 32, dtype=torch.bfloat16), torch.zeros(32)]
    outs = [torch.zeros(64, 32, dtype=torch.bfloat16), torch.zeros(32), torch.zeros(32)]
    p.check_io(ins, outs, device=False)
    with pytest.raises(ValueError, match="dtype"):
        p.check_io([ins[0].float()] + ins[1:], outs, device=False)
    with pytest.raises(ValueError, match="contiguous"):
        p.check_io([torch.zeros(32, 64, dtype=torch.bfloat16).t()] + ins[1:], outs, device=False)
    with pytest.raises(ValueError, match="elements"):
        p.check_io(ins, [torch.zeros(63, 32, dtype=torch.bfloat16)] + outs[1:], device=False)
    with pytest.raises(ValueError, match="inputs"):
        p.check_io(ins[:2], outs, device=False)
    with pytest.raises(ValueError, match="CUDA"):
        p.check_io(ins, outs)


def test_set_mask_binds_an_existing_lengths_input():
    """SURVEY 8(b)'s two-step mask: astitch_graph_input(LENGTHS, I32) then
    astitch_graph_set_mask; an unbound LENGTHS input is rejected at plan time."""
    def graph(bind):
        g = A.Graph()
        x = g.input("FULL", "BF16")
        L = g.input("LENGTHS", "I32")
        if bind:
            g.set_mask(L, 8)
        m = g.reduce("RMAX", "ROW", x)
        g.output(g.binary("SUB", x, g.broadcast("ROW", m)), "BF16")
        return g, L
    g, L = graph(True)
    p = A.Plan(g, 64, 128, device=-1, flags=A.FLAG_NO_COMPILE)
    assert p.inputs == [("FULL", "BF16"), ("LENGTHS", "I32")]
    with pytest.raises(A.AstitchError) as e:
        g.set_mask(L, 8)                                   # already has a mask
    assert e.value.status == 2
    g2, _ = graph(False)
    with pytest.raises(A.AstitchError) as e:
        A.Plan(g2, 64, 128, device=-1, flags=A.FLAG_NO_COMPILE)
    assert e.value.status == 2 and "set_mask" in _lib.lib.astitch_last_error().decode()
    g3 = A.Graph()
    x = g3.input("FULL", "F32")
    with pytest.raises(A.AstitchError) as e:
        g3.set_mask(x, 8)                                  # not a LENGTHS input
    assert e.value.status == 2
    with pytest.raises(A.AstitchError):
        g3.input("LENGTHS", "F32")                         # LENGTHS are int32


def test_tuning_string_overrides_and_errors():
    """astitch_plan_ex: explicit planner overrides (the library reads no
    environment variables); unknown keys / non-integers are argument errors."""
    spec = specs.get("C2", rows=4096)
    base = A.Plan(A.Graph.from_spec(spec), 4096, 768, device=-1, flags=A.FLAG_NO_COMPILE).describe()
    t = A.Plan(A.Graph.from_spec(spec), 4096, 768, device=-1, flags=A.FLAG_NO_COMPILE,
               tune={"threads": 256, "unroll": 2}).describe()
    assert base["tuning"] == "" and t["tuning"] == "threads=256,unroll=2"
    assert t["mapping"]["threads"] == 256 and t["mapping"]["row_unroll"] == 2
    assert base["mapping"]["threads"] != 256 or base["mapping"]["row_unroll"] != 2
    for bad in ("nope=1", "threads=abc", "threads"):
        with pytest.raises(A.AstitchError) as e:
            A.Plan(A.Graph.from_spec(spec), 4096, 768, device=-1, flags=A.FLAG_NO_COMPILE, tune=bad)
        assert e.value.status == 1
    s = A.Plan(A.Graph.from_spec(specs.get("C1", rows=4, cols=512)), 4, 512, device=-1,
               flags=A.FLAG_NO_COMPILE, tune="stream=1").describe()
    assert s["mapping"]["template"] == "row_stream"


def test_library_reads_no_planning_environment_variables():
    """A plan is a pure function of (graph, desc, tuning): no getenv in the
    planner or code generator (only the dlopen paths of libnccl / libnvrtc)."""
    src = os.path.join(ROOT, "paper_conf_asplos_zhengyzlzzzlyzs22_b200", "csrc")
    for f in ("planner.cpp", "codegen.cpp", "runtime.cpp", "graph.cpp"):
        assert "getenv" not in open(os.path.join(src, f)).read(), f


def test_disk_cubin_cache_and_plan_time(tmp_path):
    """The on-disk cubin cache: a fresh process-level miss compiles with NVRTC
    and stores the cubin; a plan of the same source in a NEW process loads it
    from disk (no NVRTC); describe() reports the plan (JIT) time split."""
    import subprocess
    import sys
    code = ("import sys, json; sys.path.insert(0, %r)\n"
            "import paper_conf_asplos_zhengyzlzzzlyzs22_b200 as A\n"
            "from workloads import specs\n"
            "A.set_cache_dir(%r)\n"
            "s = specs.get('C4', rows=5000)\n"
            "d = A.Plan(A.Graph.from_spec(s), 5000, 36, device=-1).describe()\n"
            "print(json.dumps(d['plan_time_ms']))\n") % (ROOT, str(tmp_path))
    runs = [json.loads(subprocess.run([sys.executable, "-c", code], capture_output=True, text=True,
                                      check=True).stdout.strip().splitlines()[-1]) for _ in range(2)]
    assert runs[0]["nvrtc_compiles"] >= 1 and runs[0]["cache_hits_disk"] == 0
    assert runs[1]["nvrtc_compiles"] == 0 and runs[1]["cache_hits_disk"] >= 1
    assert any(f.suffix == ".cubin" for f in tmp_path.iterdir())
    for k in ("analyse_map", "codegen", "nvrtc", "load", "total"):
        assert runs[0][k] >= 0
    assert runs[1]["nvrtc"] < runs[0]["nvrtc"]
    # a corrupted cache file is ignored (recompiled), never trusted
    for f in tmp_path.iterdir():
        f.write_bytes(b"garbage")
    r3 = json.loads(subprocess.run([sys.executable, "-c", code], capture_output=True, text=True,
                                   check=True).stdout.strip().splitlines()[-1])
    assert r3["nvrtc_compiles"] >= 1


def test_documented_tuning_keys_are_accepted():
    """Every key astitch.h documents for astitch_plan_ex parses; an unknown
    key is ERR_INVALID_ARGUMENT (keeps the header and the parser in step)."""
    import os
    import re
    hdr = open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "include", "astitch.h")).read()
    doc = hdr[hdr.index("keys: threads"):hdr.index("Values\n * a template cannot use")]
    keys = {k for k in re.findall(r"\b([a-z_]+)\b(?=[ ,(.]|$)", doc.replace("\n *", " "))
            if k in {"threads", "unroll", "team", "bps", "vec_bytes", "hoist", "tile_stages", "tile_rows", "tile_threads",
                     "split", "split_threads", "stream", "stage", "stage_kb", "portable_clusters", "sync", "prefetch",
                     "persistent", "waves", "remat", "tma", "tma_rows", "tma_stages", "tma_teams", "tma_team"}}
    assert len(keys) == 25, sorted(keys)
    spec = specs.get("C5", rows=64, cols=32)
    for k in sorted(keys):
        A.Plan(A.Graph.from_spec(spec), 64, 32, device=-1, flags=A.FLAG_NO_COMPILE, tune=f"{k}=1")
    with pytest.raises(A.AstitchError):
        A.Plan(A.Graph.from_spec(spec), 64, 32, device=-1, flags=A.FLAG_NO_COMPILE, tune="dyn_colred_rows=16")
