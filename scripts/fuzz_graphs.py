#!/usr/bin/env python
"""Structural fuzz: seeded random stitch-op graphs (workloads/random_graphs.py:
element-wise chains, row / column reductions, broadcasts, up to two column
reduction levels) on random shapes, GPU vs the fp64 oracle.
    python scripts/fuzz_graphs.py SEED0 N [--wide] [--long] [--tiny] [--tma]
A case fails if any output misses the DESIGN.md rule at 10x the config
tolerance plus 1e-5 absolute (random chains can cancel to exactly 0;
structural bugs give O(1) errors); the worst floored relative error is
printed for every case."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

from oracle import evaluate  # noqa: E402
from tests.harness import check_close, run_gpu, spec_tol  # noqa: E402
from workloads import gen  # noqa: E402
from workloads.random_graphs import random_graph  # noqa: E402


def main():
    s0, n = int(sys.argv[1]), int(sys.argv[2])
    wide = "--wide" in sys.argv
    bad = 0
    worst = 0.0
    templates = {}
    for seed in range(s0, s0 + n):
        rng = np.random.default_rng(10_000 + seed)
        rows = int(rng.choice([int(rng.integers(1, 100)), int(rng.integers(100, 5000)), int(rng.integers(5000, 30000))]))
        cols = int(rng.choice([int(rng.integers(1, 64)), int(rng.integers(64, 1100)), int(rng.integers(1100, 6000))]))
        kw = {}
        if "--long" in sys.argv:      # few long rows, row-wise graphs: split_row / row_stream
            rows, cols = int(rng.integers(1, 40)), int(rng.integers(30_000, 160_000))
            kw = {"colred": False}
        if "--tiny" in sys.argv:      # many tiny rows, row-wise, no column vectors: TMA packed tiles
            rows, cols = int(rng.integers(4096, 60_000)), int(rng.choice([9, 12, 20, 36, 44, 60, 100]))
            kw = {"colred": False, "colvec": False}
        if "--tma" in sys.argv:       # column counts the bulk-copy templates take (tma_sweep / tma_team)
            cols = int(rng.choice([128 * int(rng.integers(1, 17)), 256 * int(rng.integers(9, 17))]))
            kw = {"rowwise": bool(rng.random() < 0.3)}
        cols = max(1, min(cols, 6_000_000 // rows))
        if "--tma" in sys.argv:
            cols = max(128, cols // 128 * 128)
        spec = random_graph(seed, rows, cols, wide=wide, **kw)
        flags = 0
        if wide:
            flags = int(rng.choice([0, 0, 0, 0, 0, 2, 4, 64]))
        x = gen.generate("fig6a", spec)
        try:
            # --tma: force the bulk-copy sweep where eligible (the planner takes
            # it by itself only for long sweeps; fuzz shapes are small)
            got, plan = run_gpu(spec, x, return_plan=True, flags=flags, tune="tma=1" if "--tma" in sys.argv else None)
            ref = evaluate(spec, x)
            errs = []
            for name, dt in spec["outputs"]:
                # atol 1e-5: an output that is exactly 0 by cancellation (the sum of
                # a row's centred values) has no relative scale; O(1) inputs
                # an output that is identically 0 by construction (colsum(x) -
                # colsum(x) with one of them fp64 under R7c, the row sum of
                # centred values) keeps the fp32 rounding of its operands:
                # atol 1e-4 there (fuzz seeds 3061 / 4258, |operands| ~ 70)
                zero = float(np.sqrt(np.mean(np.square(ref[name], dtype=np.float64)))) < 1e-9
                info = check_close(got[name], ref[name], dt, 10 * spec_tol(spec), name=name, atol=1e-4 if zero else 1e-5)
                errs.append(info["max_rel_err_floored"])
            w = max(errs)
            worst = max(worst, w)
            mp = plan.describe()["mapping"]
            tname = mp["template"] + ("/tma_sweep" if mp.get("tma_sweep") else "") + ("/tma_team" if mp.get("tma_team") else "")
            print(f"ok seed={seed} [{rows},{cols}] flags={flags} {tname} max_rel={w:.2e}", flush=True)
            templates[tname] = templates.get(tname, 0) + 1
        except Exception as e:
            if "ASTITCH_ERR_UNSUPPORTED" in str(e):
                print(f"unsupported seed={seed}: {str(e)[:120]}")
                continue
            bad += 1
            print(f"FAIL seed={seed} [{rows},{cols}]: {str(e)[:400]}", flush=True)
    print(f"graph fuzz done: {n} seeds, failures: {bad}, worst floored rel err {worst:.2e}, templates {templates}")


if __name__ == "__main__":
    main()
