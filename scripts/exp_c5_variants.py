#!/usr/bin/env python
"""Where C5's time goes: the stitched kernel on C5's shapes with pieces
removed (transcendental GELU', the column reduction), CUDA-graph timed,
against the same traffic through torch.add (2 reads : 1 write)."""
import copy
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_asplos_zhengyzlzzzlyzs22_b200 as A  # noqa: E402
from workloads import specs  # noqa: E402


def timed(fn, n=10):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for _ in range(n):
            fn()
    g.replay()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    g.replay()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) * 1e3 / n


def variant(name, ops, outputs, flags=0):
    s = copy.deepcopy(specs.get("C5"))
    s["ops"], s["outputs"] = ops, outputs
    R, C = s["rows"], s["cols"]
    p = A.Plan(A.Graph.from_spec(s), R, C, device=0, flags=flags)
    ins = [torch.randn(R, C, device="cuda").to(torch.bfloat16), torch.randn(R, C, device="cuda").to(torch.bfloat16),
           torch.randn(C, device="cuda")]
    live = [i for i, (n, _, _) in enumerate(s["inputs"]) if p.inputs and True]
    ins = ins[: len(p.inputs)]
    outs = p.alloc_outputs()
    ws = p.alloc_workspace()
    us = timed(lambda: p.run(ins, outs, ws=ws))
    nbytes = sum(t.numel() * t.element_size() for t in ins) + sum(t.numel() * t.element_size() for t in outs)
    m = p.describe()["mapping"]
    print(f"{name}: {us:.1f} us, {nbytes / us / 1e3:.1f} GB/s, template {m['template']}, grid {m['grid']}, "
          f"threads {m['threads']}, regs {p.describe()['kernels'][0]['regs']}", flush=True)
    del ins, outs, ws, p
    torch.cuda.empty_cache()


def main():
    c5 = specs.get("C5")
    try:
        variant("C5 (GELU' + col sum + b_new)", c5["ops"], c5["outputs"])
    except Exception as e:
        print("C5 failed:", str(e)[:200])
    variant("mul + col sum + b_new (no GELU')",
            [("dz", "binary", "MUL", "dy", "z")] + c5["ops"][2:], c5["outputs"])
    variant("GELU' only (no col sum)", c5["ops"][:2], [("dz", "BF16")])
    variant("mul only", [("dz", "binary", "MUL", "dy", "z")], [("dz", "BF16")])
    n = 1 << 30
    x = torch.randn(n, device="cuda").to(torch.bfloat16)
    y = torch.randn(n, device="cuda").to(torch.bfloat16)
    z = torch.empty_like(x)
    us = timed(lambda: torch.add(x, y, out=z))
    print(f"torch.add: {us:.1f} us, {3 * 2 * n / us / 1e3:.1f} GB/s")


if __name__ == "__main__":
    main()
