#!/usr/bin/env python
"""Parity fuzz over seeded random shapes, offsets and ablation flags (GPU vs
the fp64 oracle):
    python scripts/fuzz_shapes.py SEED0 NSEEDS
Covers C1-C5, Fig. 5/6a/7(a), BatchNorm, remote stitching; wide rows (column
slabs), light rows (non-persistent grids), means far from the spread (R7b /
R7c), and the FORCE_GLOBAL / NO_PACK / NO_PREFETCH / NO_TMA ablations."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

from oracle import evaluate  # noqa: E402
from tests.harness import check_close, run_gpu, spec_tol  # noqa: E402
from workloads import gen, specs  # noqa: E402

FLAGS = [0, 0, 0, 0, 2, 4, 64, 32]   # mostly defaults; FORCE_GLOBAL, NO_PACK, NO_PREFETCH, NO_TMA


def main():
    s0, n = int(sys.argv[1]), int(sys.argv[2])
    bad = cases = 0
    for seed in range(s0, s0 + n):
        rng = np.random.default_rng(seed)
        for cfg in ["C1", "C2", "C3", "C4", "C5", "fig7a", "bn", "fig5", "remote", "fig6a"]:
            rows = int(rng.choice([int(rng.integers(1, 64)), int(rng.integers(64, 6000)), int(rng.integers(6000, 40000))]))
            cols = int(rng.choice([int(rng.integers(1, 128)), int(rng.integers(128, 1100)), int(rng.integers(1100, 9000))]))
            if cfg in ("C5", "fig6a") and rng.random() < 0.25:      # wide rows: column slabs / streamed rows
                cols = int(rng.integers(16384, 70000))
            cols = max(1, min(cols, 8_000_000 // max(rows, 1)))
            try:
                spec = specs.get(cfg, rows=rows, cols=cols)
            except Exception as e:  # a spec with a fixed shape
                print("skip", cfg, e)
                continue
            if spec.get("mask"):
                spec["mask"]["rows_per_segment"] = int(rng.integers(1, 300))
            flags = int(rng.choice(FLAGS))
            x = gen.generate(cfg, spec)
            if cfg in ("bn", "C4") and rng.random() < 0.3:          # means far from the spread
                k = spec["inputs"][0][0]
                x[k] = (float(rng.choice([1e3, -3e4])) + 0.01 * x[k].astype(np.float64)).astype(np.float32)
            cases += 1
            try:
                got, plan = run_gpu(spec, x, return_plan=True, flags=flags)
                ref = evaluate(spec, x)
                for name, dt in spec["outputs"]:
                    check_close(got[name], ref[name], dt, spec_tol(spec), name=f"{cfg}:{name}")
            except Exception as e:
                if "ASTITCH_ERR_UNSUPPORTED" in str(e):
                    continue
                bad += 1
                print(f"FAIL seed={seed} {cfg} rows={rows} cols={cols} flags={flags}: {str(e)[:300]}", flush=True)
    print(f"fuzz done: {cases} cases, failures: {bad}")


if __name__ == "__main__":
    main()
