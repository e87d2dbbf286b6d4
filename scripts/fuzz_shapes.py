#!/usr/bin/env python
"""One-off parity fuzz over seeded random shapes (GPU vs the fp64 oracle):
    python scripts/fuzz_shapes.py SEED0 NSEEDS"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

from oracle import evaluate  # noqa: E402
from tests.harness import check_close, run_gpu, spec_tol  # noqa: E402
from workloads import gen, specs  # noqa: E402


def main():
    s0, n = int(sys.argv[1]), int(sys.argv[2])
    bad = 0
    for seed in range(s0, s0 + n):
        rng = np.random.default_rng(seed)
        for cfg in ["C1", "C2", "C3", "C4", "C5", "fig7a", "bn", "fig5", "remote"]:
            rows = int(rng.choice([int(rng.integers(1, 64)), int(rng.integers(64, 6000)), int(rng.integers(6000, 40000))]))
            cols = int(rng.choice([int(rng.integers(1, 128)), int(rng.integers(128, 1100)), int(rng.integers(1100, 9000))]))
            cols = max(1, min(cols, 8_000_000 // rows))
            try:
                spec = specs.get(cfg, rows=rows, cols=cols)
            except Exception as e:  # a spec with a fixed shape
                print("skip", cfg, e)
                continue
            if spec.get("mask"):
                spec["mask"]["rows_per_segment"] = int(rng.integers(1, 300))
            x = gen.generate(cfg, spec)
            try:
                got, plan = run_gpu(spec, x, return_plan=True)
                ref = evaluate(spec, x)
                for name, dt in spec["outputs"]:
                    check_close(got[name], ref[name], dt, spec_tol(spec), name=f"{cfg}:{name}")
            except Exception as e:
                bad += 1
                print(f"FAIL seed={seed} {cfg} rows={rows} cols={cols}: {str(e)[:300]}", flush=True)
    print("fuzz done, failures:", bad)


if __name__ == "__main__":
    main()
