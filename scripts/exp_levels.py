#!/usr/bin/env python
"""Per-level cost of multi-level global sweeps: times graphs that add one
barrier level at a time (column sum only -> centred second moment -> full
BatchNorm) under tuning overrides, fp32 [R, C] on cuda:0, CUDA events, L2
flushed between iterations.
    python scripts/exp_levels.py [R C] [TUNE ...]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def graphs(R):
    x = [("x", "FULL", "F32")]
    base = [("s1", "reduce", "SUM", "COL", "x"), ("n", "const", float(R)), ("mean", "binary", "DIV", "s1", "n")]
    cen = base + [("mb", "broadcast", "COL", "mean"), ("xc", "binary", "SUB", "x", "mb")]
    var = cen + [("xc2", "binary", "MUL", "xc", "xc"), ("s2", "reduce", "SUM", "COL", "xc2"),
                 ("var", "binary", "DIV", "s2", "n")]
    norm = var + [("eps", "const", 1e-5), ("ve", "binary", "ADD", "var", "eps"), ("rs", "unary", "RSQRT", "ve"),
                  ("rb", "broadcast", "COL", "rs"), ("y", "binary", "MUL", "xc", "rb")]
    return {
        "copy": ({"ops": [("two", "const", 2.0), ("y", "binary", "MUL", "x", "two")], "outputs": [("y", "F32")]}, 8),
        "colsum": ({"ops": base, "outputs": [("mean", "F32")]}, 4),
        "center": ({"ops": cen, "outputs": [("xc", "F32"), ("mean", "F32")]}, 12),
        "var": ({"ops": var, "outputs": [("var", "F32")]}, 8),
        "bn": ({"ops": norm, "outputs": [("y", "F32"), ("var", "F32")]}, 16),
    }, x


def main():
    import torch
    import paper_conf_asplos_zhengyzlzzzlyzs22_b200 as A
    args = sys.argv[1:]
    R, C = 1048576, 1024
    if len(args) >= 2 and args[0].isdigit():
        R, C, args = int(args[0]), int(args[1]), args[2:]
    tunes = [None if t == "-" else t for t in args] or [None]
    gs, ins_spec = graphs(R)
    x = torch.randn(R, C, device="cuda")
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    only = os.environ.get("EXP_GRAPHS")
    for name, (g, bpe) in gs.items():
        if only and name not in only.split(","):
            continue
        for tune in tunes:
            spec = {"name": name, "rows": R, "cols": C, "inputs": ins_spec, "mask": None, **g}
            try:
                p = A.Plan(A.Graph.from_spec(spec), R, C, device=0, tune=tune)
            except Exception as e:
                print(f"{name:7s} {tune!s:28s} plan failed: {str(e)[:100]}")
                continue
            outs, ws = p.alloc_outputs(), p.alloc_workspace()
            for _ in range(3):
                p.run([x], outs, ws=ws)
            ts = []
            for _ in range(10):
                flush.zero_()
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record()
                p.run([x], outs, ws=ws)
                b.record()
                torch.cuda.synchronize()
                ts.append(a.elapsed_time(b))
            ts.sort()
            ms = ts[len(ts) // 2]
            m = p.describe()["mapping"]
            k = p.describe()["kernels"][0]
            print(f"{name:7s} {tune!s:28s} {ms * 1e3:9.1f} us  {bpe * R * C / ms / 1e6:7.1f} GB/s(compulsory-ish)  "
                  f"{m['template']} thr {k['threads']} grid {k['grid']} regs {k['regs']} spill {k['spill_bytes']} "
                  f"team {m['team']} rpb {m['rows_per_block']} unroll {m['row_unroll']} pf {m['prefetch']} "
                  f"sync {m['sync_steps']}", flush=True)


if __name__ == "__main__":
    main()
