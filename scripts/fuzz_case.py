#!/usr/bin/env python
"""Rebuild one graph-fuzz case exactly as scripts/fuzz_graphs.py draws it and
compare the GPU with the oracle under several planner tunings.
    python scripts/fuzz_case.py SEED [--wide] [--tma] [--long] [--tiny] [--tune a=b ...] [--show]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

from workloads.random_graphs import random_graph  # noqa: E402


def case(seed, argv):
    wide = "--wide" in argv
    rng = np.random.default_rng(10_000 + seed)
    rows = int(rng.choice([int(rng.integers(1, 100)), int(rng.integers(100, 5000)), int(rng.integers(5000, 30000))]))
    cols = int(rng.choice([int(rng.integers(1, 64)), int(rng.integers(64, 1100)), int(rng.integers(1100, 6000))]))
    kw = {}
    if "--long" in argv:
        rows, cols = int(rng.integers(1, 40)), int(rng.integers(30_000, 160_000))
        kw = {"colred": False}
    if "--tiny" in argv:
        rows, cols = int(rng.integers(4096, 60_000)), int(rng.choice([9, 12, 20, 36, 44, 60, 100]))
        kw = {"colred": False, "colvec": False}
    if "--tma" in argv:
        cols = int(rng.choice([128 * int(rng.integers(1, 17)), 256 * int(rng.integers(9, 17))]))
        kw = {"rowwise": bool(rng.random() < 0.3)}
    cols = max(1, min(cols, 6_000_000 // rows))
    if "--tma" in argv:
        cols = max(128, cols // 128 * 128)
    spec = random_graph(seed, rows, cols, wide=wide, **kw)
    flags = int(rng.choice([0, 0, 0, 0, 0, 2, 4, 64])) if wide else 0
    return spec, flags


def main():
    seed = int(sys.argv[1])
    spec, flags = case(seed, sys.argv)
    tunes = [a.split("=", 1)[1] for a in sys.argv if a.startswith("--tune=")] or ["tma=1" if "--tma" in sys.argv else None]
    if "--show" in sys.argv:
        import json
        print(json.dumps(spec, indent=0)[:4000])
        print("flags", flags)
        return
    from oracle import evaluate
    from tests.harness import check_close, run_gpu, spec_tol
    from workloads import gen
    x = gen.generate("fig6a", spec)
    ref = evaluate(spec, x)
    for t in tunes:
        got, plan = run_gpu(spec, x, return_plan=True, flags=flags, tune=t)
        m = plan.describe()["mapping"]
        print(f"tune={t} template={m['template']} tma_sweep={m['tma_sweep']} tma_team={m['tma_team']}")
        for name, dt in spec["outputs"]:
            g, r = got[name], ref[name]
            err = np.abs(g - r)
            i = int(np.argmax(err))
            print(f"  {name} shape={g.shape} max_abs_err={err.max():.3e} at {np.unravel_index(i, g.shape)} gpu={g.flat[i]!r} ref={r.flat[i]!r} rms_ref={np.sqrt(np.mean(r*r)):.3e}")


if __name__ == "__main__":
    main()
