"""Runtime behaviour of the C ABI on the GPU: error codes, no-op shapes,
workspace reuse (self-resetting grid barrier), host-buffer runs, CUDA-graph
capture, concurrent plans on separate streams, measurement aids."""

import ctypes as ct

import numpy as np
import pytest

import paper_conf_asplos_zhengyzlzzzlyzs22_b200 as A
from paper_conf_asplos_zhengyzlzzzlyzs22_b200 import _lib
from oracle import evaluate
from tests.harness import check_close, device_inputs, from_torch, run_gpu, spec_tol, to_torch
from workloads import gen, specs

pytestmark = pytest.mark.gpu


def _plan(cfg, rows=None, cols=None, flags=0):
    spec = specs.get(cfg, rows=rows, cols=cols)
    return spec, A.Plan(A.Graph.from_spec(spec), spec["rows"], spec["cols"], device=0, flags=flags)


def test_rows_zero_is_noop():
    import torch
    from torch.profiler import ProfilerActivity, profile
    spec, p = _plan("C5", rows=0, cols=64)
    ins = [torch.empty((0, 64), dtype=torch.bfloat16, device="cuda"),
           torch.empty((0, 64), dtype=torch.bfloat16, device="cuda"), torch.zeros(64, device="cuda")]
    outs = p.alloc_outputs()
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        p.run(ins, outs)
        torch.cuda.synchronize()
    assert not [e for e in prof.events() if e.name.startswith("astitch_")]


def test_misaligned_and_missing_workspace():
    import torch
    spec, p = _plan("C1")
    x = torch.randn(32 * 128 + 1, device="cuda")
    y = torch.empty(32 * 128, device="cuda")
    with pytest.raises(A.AstitchError) as e:
        p.run([x[1:]], [y])                         # 4-byte offset: not 16-byte aligned
    assert e.value.status == 1 and "aligned" in str(e.value)
    spec, p5 = _plan("C5", rows=512, cols=128)
    ins = device_inputs(spec, gen.generate("C5", spec))
    outs = p5.alloc_outputs()
    ip = _lib.ptr_array([t.data_ptr() for t in ins])
    op = _lib.ptr_array([t.data_ptr() for t in outs])
    st = _lib.lib.astitch_run(p5.handle, ip, op, None, ct.c_void_p(torch.cuda.current_stream().cuda_stream))
    assert st == 1 and "workspace" in _lib.lib.astitch_last_error().decode()


def test_workspace_reuse_many_runs_barrier_self_resets():
    import torch
    spec = specs.get("C5", rows=4099, cols=256)
    x = gen.generate("C5", spec)
    p = A.Plan(A.Graph.from_spec(spec), spec["rows"], spec["cols"], device=0)
    ins, outs, ws = device_inputs(spec, x), p.alloc_outputs(), p.alloc_workspace()
    p.run(ins, outs, ws=ws)
    torch.cuda.synchronize()
    first = [from_torch(t) for t in outs]
    for _ in range(50):                              # no re-init between runs
        p.run(ins, outs, ws=ws)
    torch.cuda.synchronize()
    for a, t in zip(first, outs):
        assert np.array_equal(a, from_torch(t))
    check_close(first[1], evaluate(spec, x)["db"], "F32", spec_tol(spec), "db")


def test_run_host_matches_device_run():
    import torch
    spec = specs.get("C3", rows=2048)
    spec["mask"]["rows_per_segment"] = 256
    x = gen.generate("C3", spec)
    ref, p = run_gpu(spec, x, return_plan=True)
    host_in = [to_torch(x[n], d, None).pin_memory() for n, _, d in spec["inputs"]]
    dev_in = device_inputs(spec, x)
    dev_out = p.alloc_outputs()
    host_out = [torch.empty(t.shape, dtype=t.dtype).pin_memory() for t in dev_out]
    p.run_host(host_in, host_out, dev_in, dev_out)
    torch.cuda.synchronize()
    assert np.array_equal(from_torch(host_out[0]), ref["p"])


@pytest.mark.parametrize("cfg,rows,chunks", [("C3", 8192, 5), ("C4", 30011, 7), ("C5", 20000, 4),
                                             ("C2", 4096, 3), ("C5int", 8192, 6), ("remote", 3000, 4)])
def test_run_host_pipelined(cfg, rows, chunks):
    """Chunked host pipeline (H2D / kernel / D2H overlapped on three streams):
    row outputs bitwise equal to the one-shot run, column outputs within the
    oracle tolerance (chunk totals are accumulated in a different order)."""
    import torch
    spec = specs.get(cfg, rows=rows)
    if spec.get("mask"):
        spec["mask"]["rows_per_segment"] = 1000      # chunk boundaries fall inside segments
    x = gen.generate(cfg, spec)
    ref, p = run_gpu(spec, x, return_plan=True)
    oracle = evaluate(spec, x)
    host_in = [to_torch(x[n], d, None).pin_memory() for n, _, d in spec["inputs"]]
    dev_in = [torch.empty_like(h, device="cuda") for h in host_in]
    dev_out = p.alloc_outputs()
    host_out = [torch.empty(t.shape, dtype=t.dtype).pin_memory() for t in dev_out]
    for _ in range(2):                                # second call reuses streams / chunk kernels
        p.run_host(host_in, host_out, dev_in, dev_out, chunks=chunks)
        torch.cuda.synchronize()
    kinds = [k for k, _ in p.outputs]
    for (name, dt), t, k in zip(spec["outputs"], host_out, kinds):
        got = from_torch(t)
        if k == "COLVEC":
            check_close(got, oracle[name], dt, spec_tol(spec), name)
            if cfg == "C5int":
                assert np.array_equal(got, ref[name])    # integer data: exact in any order
        else:
            assert np.array_equal(got, ref[name]), name


@pytest.mark.parametrize("cfg", ["C3", "C5", "C4"])
def test_cuda_graph_capture(cfg):
    import torch
    spec = specs.get(cfg, rows=8192)
    if spec.get("mask"):
        spec["mask"]["rows_per_segment"] = 1024
    x = gen.generate(cfg, spec)
    ref, p = run_gpu(spec, x, return_plan=True)
    ins, outs, ws = device_inputs(spec, x), p.alloc_outputs(), p.alloc_workspace()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        p.run(ins, outs, ws=ws)
    for _ in range(3):
        g.replay()
    torch.cuda.synchronize()
    for (name, _), t in zip(spec["outputs"], outs):
        assert np.array_equal(from_torch(t), ref[name]), name


def test_two_plans_two_streams_concurrently():
    import torch
    s5 = specs.get("C5", rows=20000, cols=512)
    s3 = specs.get("C3", rows=8192)
    s3["mask"]["rows_per_segment"] = 1024
    x5, x3 = gen.generate("C5", s5), gen.generate("C3", s3)
    r5, p5 = run_gpu(s5, x5, return_plan=True)
    r3, p3 = run_gpu(s3, x3, return_plan=True)
    st_a, st_b = torch.cuda.Stream(), torch.cuda.Stream()
    i5, o5, w5 = device_inputs(s5, x5), p5.alloc_outputs(), p5.alloc_workspace()
    i3, o3 = device_inputs(s3, x3), p3.alloc_outputs()
    torch.cuda.synchronize()
    for _ in range(5):
        p5.run(i5, o5, ws=w5, stream=st_a)
        p3.run(i3, o3, stream=st_b)
    torch.cuda.synchronize()
    for (name, _), t in zip(s5["outputs"], o5):
        assert np.array_equal(from_torch(t), r5[name])
    assert np.array_equal(from_torch(o3[0]), r3["p"])


def test_bench_copy_and_barrier_aids():
    import torch
    src = torch.randint(0, 255, (1 << 20,), dtype=torch.uint8, device="cuda")
    dst = torch.zeros_like(src)
    A.bench_copy(0, src, dst, src.numel())
    torch.cuda.synchronize()
    assert torch.equal(src, dst)
    ws = torch.zeros(64, dtype=torch.int32, device="cuda")
    for blocks in (1, 37, 148, 296):
        A.bench_barrier(0, blocks, 256, 10, ws)
    torch.cuda.synchronize()
    assert int(ws[0].item()) == 0                    # arrival counter returns to 0


def test_sharded_world1_equals_run():
    from paper_conf_asplos_zhengyzlzzzlyzs22_b200.dist import ShardedPlan
    spec = specs.get("C5", rows=3000, cols=256)
    x = gen.generate("C5", spec)
    ref = run_gpu(spec, x)
    sp = ShardedPlan(A.Graph.from_spec(spec), 3000, 256, 1, 0, 0)
    ins, outs = device_inputs(spec, x), sp.plan.alloc_outputs()
    sp.run(ins, outs)
    import torch
    torch.cuda.synchronize()
    for (name, _), t in zip(spec["outputs"], outs):
        assert np.array_equal(from_torch(t), ref[name])


def test_peer_exchange_misuse_errors():
    import torch
    """astitch_peer_* / astitch_run_fused argument checks (ERR_INVALID_ARGUMENT)."""
    import paper_conf_asplos_zhengyzlzzzlyzs22_b200 as A
    from paper_conf_asplos_zhengyzlzzzlyzs22_b200.dist import PeerExchange, ShardedPlan
    from workloads import specs
    spec = specs.get("C5", rows=1000, cols=64)
    g = A.Graph.from_spec(spec)
    s0, s1 = ShardedPlan(g, 1000, 64, 2, 0, 0), ShardedPlan(g, 1000, 64, 2, 1, 0)
    x0, x1 = PeerExchange(s0.plan), PeerExchange(s1.plan)
    with pytest.raises(A.AstitchError):
        x0.link(0, x1)                    # x1 is rank 1, not 0
    with pytest.raises(A.AstitchError):
        x0.link(5, x1)                    # rank out of range
    ins = [torch.zeros(s0.row_count, 64, dtype=torch.bfloat16, device="cuda"),
           torch.zeros(s0.row_count, 64, dtype=torch.bfloat16, device="cuda"), torch.zeros(64, device="cuda")]
    s0.peer = x0
    with pytest.raises(A.AstitchError):   # peer 1 not mapped yet
        s0.run(ins, s0.plan.alloc_outputs())
    other = ShardedPlan(A.Graph.from_spec(specs.get("C5", rows=1000, cols=128)), 1000, 128, 2, 1, 0)
    with pytest.raises(A.AstitchError):   # different plan (cols): buffer sizes differ
        x0.link(1, PeerExchange(other.plan))


@pytest.mark.parametrize("cfg,rows,cols", [("C1", None, None), ("C5", 4099, 256), ("C3", 1024, None)])
def test_bind_matches_run(cfg, rows, cols):
    """Plan.bind(): the pre-marshalled eager call computes what run() does
    (bitwise: same kernel, same buffers layout), repeatedly."""
    import torch
    spec = specs.get(cfg, rows=rows, cols=cols)
    if spec.get("mask"):
        spec["mask"]["rows_per_segment"] = 256
    x = gen.generate(cfg, spec)
    p = A.Plan(A.Graph.from_spec(spec), spec["rows"], spec["cols"], device=0)
    ins = device_inputs(spec, x)
    o1, o2 = p.alloc_outputs(), p.alloc_outputs()
    p.run(ins, o1)
    f = p.bind(ins, o2)
    for _ in range(3):
        f()
    torch.cuda.synchronize()
    for a, b in zip(o1, o2):
        assert torch.equal(a, b)
    ref = evaluate(spec, x)
    for (name, dt), t in zip(spec["outputs"], o2):
        check_close(from_torch(t), ref[name], dt, spec_tol(spec), name=f"{cfg}:{name}")
