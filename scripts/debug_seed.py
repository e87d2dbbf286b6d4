#!/usr/bin/env python
"""Run one random-graph fuzz case on the GPU and print where it differs from
the oracle (rows / columns of the worst elements).
    python scripts/debug_seed.py SEED ROWS COLS"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

from oracle import evaluate  # noqa: E402
from tests.harness import run_gpu  # noqa: E402
from workloads import gen  # noqa: E402
from workloads.random_graphs import random_graph  # noqa: E402


def main():
    seed, rows, cols = (int(a) for a in sys.argv[1:4])
    spec = random_graph(seed, rows, cols)
    x = gen.generate("fig6a", spec)
    got, plan = run_gpu(spec, x, return_plan=True)
    ref = evaluate(spec, x)
    print("mapping", {k: plan.describe()["mapping"][k] for k in ("template", "team", "chunks_per_lane", "vec_elems",
                                                                 "threads", "grid", "row_unroll", "prefetch")})
    for name, _ in spec["outputs"]:
        g, r = got[name], ref[name]
        err = np.abs(g - r)
        s = float(np.sqrt(np.mean(r * r))) or 1.0
        bad = err > 1e-3 * np.maximum(np.abs(r), s)
        print(name, g.shape, "bad", int(bad.sum()))
        if bad.any():
            idx = np.argwhere(bad)
            print("  first bad", idx[:10].tolist())
            if g.ndim == 2:
                print("  bad rows", np.unique(idx[:, 0])[:20].tolist(), "bad cols", np.unique(idx[:, 1])[:20].tolist())
            i = tuple(idx[0])
            print("  gpu", g[i], "ref", r[i])


if __name__ == "__main__":
    main()
