#!/usr/bin/env python
"""Redundancy check from ncu source pages (SURVEY 8(c) "performance claims"):
the MUFU (transcendental) thread-instructions a stitched kernel executed vs
the count the op-by-op definition needs, one per heavy op per element (plus
the row-scalar ops every lane of a team computes).  A ratio near 1 means every
heavy element-wise op ran once per element (element/operator-level reuse,
P:L194-L196): no producer was recomputed for its consumers.

    python scripts/mufu_evidence.py [gpurun_out] [round] > profiles/<round>_mufu.md
"""
import csv
import io
import os
import subprocess
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

from workloads import gen, specs  # noqa: E402


def mufu_counts(rep):
    r = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                       capture_output=True, text=True)
    rows = list(csv.reader(io.StringIO(r.stdout)))
    h = rows[1]
    src, th = h.index("Source"), h.index("Thread Instructions Executed")
    pr = h.index("Predicated-On Thread Instructions Executed")
    out = {}
    for row in rows[2:]:
        t = row[src].strip().split()
        if not t:
            continue
        op = t[1] if t[0].startswith("@") else t[0]
        if op.startswith("MUFU"):
            out[op] = out.get(op, 0) + int(row[pr] or row[th])
    return out


def expected(cfg):
    """(expected MUFU thread-ops, how it is counted)."""
    if cfg == "C5":
        R, C = 1_048_576, 1024
        return 2 * R * C, "GELU' sigma form: 1 ex2 + 1 rcp per element"
    if cfg == "C2":
        R, C, T = 4096, 768, 32
        return 2 * R * C + R * T, "GELU sigma form: ex2 + rcp per element; rsqrt per row on each of 32 lanes"
    if cfg == "C4":
        return 2_000_000, "rsqrt per row (thread per row)"
    if cfg == "C3":
        s = specs.get("C3")
        L = gen.lengths_for(s, 3).astype(np.int64)
        T, E = 16, 8
        comp = ((L + T * E - 1) // (T * E)) * T * E   # chunk-uniform skipping: whole team chunks
        return int((comp * 8192).sum() + 524288 * T), \
            "ex2 per element of every team chunk holding a valid column (128 columns); rcp per row per lane"
    if cfg == "C3v":
        s = gen.ragged_spec(specs.get("C3v"), 3)
        T, E, V = 8, 8, 8
        tot = 0
        for r, c in zip(s["segments"]["seg_rows"], s["segments"]["seg_cols"]):
            kf = min(c // (T * E), V)
            live = min(kf + 1, V) * T * E
            tot += r * (live + T)
        return tot, "ex2 per element of chunks 0..KF (KF specialisation, 64 columns); rcp per row per lane"
    return None, ""


def main(out="gpurun_out", rnd=""):
    print("# MUFU (transcendental) thread-instructions: executed vs needed (ncu source page)\n")
    print("| cfg | executed | by opcode | needed | ratio | counted as |")
    print("|---|---|---|---|---|---|")
    for cfg in ("C2", "C3", "C4", "C5", "C3v"):
        rep = os.path.join(out, f"prof_{rnd}_{cfg}.ncu-rep" if rnd else f"prof_{cfg}.ncu-rep")
        if not os.path.exists(rep):
            continue
        got = mufu_counts(rep)
        tot = sum(got.values())
        need, how = expected(cfg)
        ratio = f"{tot / need:.3f}" if need else "-"
        print(f"| {cfg} | {tot:,} | {', '.join(f'{k} {v:,}' for k, v in sorted(got.items()))} | "
              f"{need:,} | {ratio} | {how} |")


if __name__ == "__main__":
    main(*(sys.argv[1:3]))
