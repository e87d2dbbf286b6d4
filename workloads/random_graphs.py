"""Seeded random stitch-op graphs (DATA ONLY: specs in the workloads/specs.py
format) for structural fuzzing of the planner and code generator against the
oracle.  Values stay bounded (inputs N(0,1); EXP / LOG / SQRT / RSQRT / RCP /
DIV only on bounded or shifted-positive operands) so fp32 rounding, not
overflow, is the only difference the oracle comparison can see."""

from __future__ import annotations

import numpy as np

SAFE_UNARY = ["NEG", "ABS", "TANH", "SIGMOID", "GELU_TANH", "ERF", "GELU_TANH_GRAD"]
BINARY = ["ADD", "SUB", "MUL", "MAX", "MIN"]


def random_graph(seed: int, rows: int, cols: int, n_ops: int | None = None, wide: bool = False,
                 colred: bool = True, colvec: bool = True, rowwise: bool = True) -> dict:
    """wide=True: also random F16 inputs, BF16 / F16 outputs and key-padding
    masks (the "wide" fuzz); False keeps the round-2 regression seeds stable.
    rowwise=False: no ROWVEC input and column reductions only (the one-sweep
    graphs tma_sweep takes)."""
    rng = np.random.default_rng(seed)
    ops, inputs = [], []
    vals = {"FULL": [], "ROWVEC": [], "COLVEC": []}
    nfull = int(rng.integers(1, 4))
    for i in range(nfull):
        n = f"x{i}"
        inputs.append((n, "FULL", str(rng.choice(["F32", "BF16", "F16"] if wide else ["F32", "BF16"]))))
        vals["FULL"].append(n)
    if rng.random() < 0.5 and rowwise:
        inputs.append(("rv", "ROWVEC", "F32"))
        vals["ROWVEC"].append("rv")
    if rng.random() < 0.5 and colvec:
        inputs.append(("cv", "COLVEC", "F32"))
        vals["COLVEC"].append("cv")
    k = [0]

    def new(kind):
        k[0] += 1
        n = f"v{k[0]}"
        vals[kind].append(n)
        return n

    ops.append(("one", "const", 1.0))
    ops.append(("inv_c", "const", 1.0 / cols))
    ops.append(("inv_r", "const", 1.0 / max(rows, 1)))
    ncolred = 0
    for _ in range(n_ops or int(rng.integers(4, 13))):
        choice = rng.random()
        kind = str(rng.choice([kk for kk in vals if vals[kk]]))
        a = str(rng.choice(vals[kind]))
        if choice < 0.25:                                   # unary
            op = str(rng.choice(SAFE_UNARY + ["EXP_T", "LOG1P", "SQRT1P"]))
            if op == "EXP_T":                               # exp(tanh(a)): bounded
                t = new(kind); ops.append((t, "unary", "TANH", a))
                ops.append((new(kind), "unary", "EXP", t))
            elif op in ("LOG1P", "SQRT1P"):                 # log / sqrt / rsqrt / rcp of |a| + 1
                t = new(kind); ops.append((t, "unary", "ABS", a))
                u = new(kind); ops.append((u, "binary", "ADD", t, "one"))
                ops.append((new(kind), "unary", str(rng.choice(["LOG", "SQRT", "RSQRT", "RCP"])), u))
            else:
                ops.append((new(kind), "unary", op, a))
        elif choice < 0.55:                                 # binary (same kind, or a broadcast into FULL)
            if kind == "FULL" and rng.random() < 0.4 and (vals["ROWVEC"] or vals["COLVEC"]):
                bk = "ROWVEC" if (vals["ROWVEC"] and (not vals["COLVEC"] or rng.random() < 0.5)) else "COLVEC"
                b0 = str(rng.choice(vals[bk]))
                b = new("FULL"); ops.append((b, "broadcast", "ROW" if bk == "ROWVEC" else "COL", b0))
            else:
                b = str(rng.choice(vals[kind]))
            op = str(rng.choice(BINARY + ["DIV1P"]))
            if op == "DIV1P":                               # a / (|b| + 1)
                t = new(kind if kind != "FULL" or b.startswith("v") else "FULL"); ops.append((t, "unary", "ABS", b))
                u = new(kind); ops.append((u, "binary", "ADD", t, "one"))
                ops.append((new(kind), "binary", "DIV", a, u))
            else:
                ops.append((new(kind), "binary", op, a, b))
        elif choice < 0.8 and vals["FULL"]:                  # reduction of a FULL value
            a = str(rng.choice(vals["FULL"]))
            axis = "ROW" if (rng.random() < 0.6 or ncolred >= 2 or not colred) else "COL"
            if not rowwise:
                if ncolred >= 2:
                    continue
                axis = "COL"
            red = str(rng.choice(["SUM", "RMAX"]))
            r = new("ROWVEC" if axis == "ROW" else "COLVEC")
            ops.append((r, "reduce", red, axis, a))
            if red == "SUM":                                # mean-like scaling
                m = new("ROWVEC" if axis == "ROW" else "COLVEC")
                ops.append((m, "binary", "MUL", r, "inv_c" if axis == "ROW" else "inv_r"))
            ncolred += axis == "COL"
        else:                                               # broadcast back into FULL and combine
            bk = "ROWVEC" if vals["ROWVEC"] and (not vals["COLVEC"] or rng.random() < 0.5) else "COLVEC"
            if not vals[bk] or not vals["FULL"]:
                continue
            b = new("FULL"); ops.append((b, "broadcast", "ROW" if bk == "ROWVEC" else "COL", str(rng.choice(vals[bk]))))
            ops.append((new("FULL"), "binary", str(rng.choice(["ADD", "SUB", "MUL"])), str(rng.choice(vals["FULL"][:-1] or vals["FULL"])), b))
    # outputs: the last value of each kind produced by an op (plus a random FULL)
    produced = [o[0] for o in ops if o[1] != "const"]
    kinds = {}
    for n, kk, _ in inputs:
        kinds[n] = kk
    for o in ops:
        if o[1] == "const":
            continue
        for kk, lst in vals.items():
            if o[0] in lst:
                kinds[o[0]] = kk
    outs = []
    for kk in ("FULL", "ROWVEC", "COLVEC"):
        cand = [n for n in produced if kinds.get(n) == kk]
        if cand:
            outs.append((cand[-1], "F32"))
    if not outs:
        outs.append((vals["FULL"][0], "F32"))
    mask = None
    if wide:
        outs = [(n, str(rng.choice(["F32", "BF16", "F16"])) if kinds.get(n) == "FULL" else "F32") for n, _ in outs]
        if rng.random() < 0.25 and colvec:
            rps = int(rng.integers(1, 200))
            inputs.append(("L", "LENGTHS", "I32"))
            mask = {"lengths": "L", "rows_per_segment": rps}
    return {"name": f"random_{seed}", "rows": rows, "cols": cols, "inputs": inputs, "mask": mask, "ops": ops,
            "outputs": outs}
