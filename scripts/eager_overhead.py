#!/usr/bin/env python
"""Host-side cost of one eager astitch_run (no CUDA graph): the Python
binding's marshalling vs the C-ABI call vs torch's own launch of a tiny
kernel.  Prints us per call for back-to-back launches on one stream."""
import ctypes as ct
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    import torch
    import paper_conf_asplos_zhengyzlzzzlyzs22_b200 as A
    from paper_conf_asplos_zhengyzlzzzlyzs22_b200._lib import lib, ptr_array
    from workloads import gen, specs
    cfg = sys.argv[1] if len(sys.argv) > 1 else "C1"
    flags = int(sys.argv[2]) if len(sys.argv) > 2 else 0
    s = specs.get(cfg)
    x = gen.generate(cfg, s)
    p = A.Plan(A.Graph.from_spec(s), s["rows"], s["cols"], device=0, flags=flags)
    from tests.harness import device_inputs
    ins = device_inputs(s, x)
    outs = p.alloc_outputs()
    ws = p.alloc_workspace()
    N = 2000

    def timeit(fn, label):
        for _ in range(50):
            fn()
        torch.cuda.synchronize()
        t = time.perf_counter()
        for _ in range(N):
            fn()
        th = time.perf_counter() - t
        torch.cuda.synchronize()
        tt = time.perf_counter() - t
        print(f"{cfg} flags={flags} {label}: host {th / N * 1e6:.2f} us/call, host+drain {tt / N * 1e6:.2f} us/call")

    timeit(lambda: p.run(ins, outs, ws=ws), "Plan.run")
    ia = ptr_array([t.data_ptr() for t in ins])
    oa = ptr_array([t.data_ptr() for t in outs])
    w = ct.c_void_p(ws.data_ptr() if ws is not None else 0)
    st = ct.c_void_p(torch.cuda.current_stream().cuda_stream)
    timeit(lambda: lib.astitch_run(p.handle, ia, oa, w, st), "astitch_run (pre-marshalled)")
    if hasattr(p, "bind"):
        f = p.bind(ins, outs, ws=ws)
        timeit(f, "Plan.bind()()")
    y = torch.empty(16, device="cuda")
    timeit(lambda: y.add_(1.0), "torch add_ (16 floats)")


if __name__ == "__main__":
    main()
