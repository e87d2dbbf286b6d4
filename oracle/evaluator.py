"""Unfused, op-by-op fp64 CPU oracle for AStitch memory-intensive subgraphs.

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py`` (its ``cpu_baseline`` leg and ``--impl reference`` arm) may import
this module.  The product path (``paper_conf_asplos_zhengyzlzzzlyzs22_b200``)
never imports, calls or links it, and it imports nothing from the product.

What it computes.  The paper states that stitching changes how a subgraph is
executed, not what it computes: "the accuracy are the same between AStitch and
other techniques" (Sec. 6.1).  So the oracle is the plain
definition of the subgraph: every op of the spec is evaluated one at a time,
in the spec's topological order, every intermediate tensor is materialised,
and all arithmetic is fp64 on the exact (widened) input values.  Nothing is
fused, reordered or rounded.

Op semantics (each is the textbook definition):

* element-wise ops apply per element (Sec. 2.1; "broadcast is often
  regarded as element-wise");
* ``reduce ROW`` reduces the contiguous (last) dimension, ``reduce COL`` the
  other one (Sec. 2.1): [R,C] -> [R] or [C];
* ``broadcast ROW`` maps [R] -> [R,C] (v[r]); ``broadcast COL`` maps [C] -> [R,C];
* a mask (reading R9) makes element (r,c) invalid iff c >= L[r // rps];
  invalid elements are absent from reductions (identity 0 for SUM, -inf for
  RMAX) and FULL outputs are 0 there.

Readings used where the paper is silent (DESIGN.md Sec. "Readings"):
R5 gelu_tanh constants sqrt(2/pi), 0.044715; R7 biased variance;
R11 integer exponents of POW are repeated multiplication; R12 RMAX propagates
NaN (numpy semantics); R14 a fully-masked reduction yields its identity.

Evaluation order: the rows are processed in chunks (memory only).  Column
reductions accumulate fp64 chunk partials in chunk order; ops that consume a
column reduction (directly or through ``broadcast COL``) are evaluated in a
later pass over the rows once every chunk has been reduced — one pass per
level of dependent column reductions (e.g. BatchNorm: mean, then variance of
the centred values), recomputing the lower-level values in each pass.  This
is the definition, split over rows; it has no blocking across columns and no
fusion.
"""

from __future__ import annotations

import math

import numpy as np
import scipy.special

GELU_C = math.sqrt(2.0 / math.pi)   # tanh-form GELU constants (reading R5)
GELU_K = 0.044715

# ----------------------------------------------------------------------------
# Element-wise op definitions (fp64)
# ----------------------------------------------------------------------------


def _gelu_tanh(x):
    """GELU, tanh approximation: 0.5 x (1 + tanh(sqrt(2/pi) (x + 0.044715 x^3)))."""
    return 0.5 * x * (1.0 + np.tanh(GELU_C * (x + GELU_K * x * x * x)))


def _gelu_tanh_grad(x):
    """d/dx of _gelu_tanh, by the product and chain rules:
    0.5 (1 + t) + 0.5 x (1 - t^2) sqrt(2/pi) (1 + 3 * 0.044715 x^2),  t = tanh(u)."""
    u = GELU_C * (x + GELU_K * x * x * x)
    t = np.tanh(u)
    return 0.5 * (1.0 + t) + 0.5 * x * (1.0 - t * t) * GELU_C * (1.0 + 3.0 * GELU_K * x * x)


def _gelu_erf(x):
    """Exact GELU: x * Phi(x) = 0.5 x (1 + erf(x / sqrt(2)))."""
    return 0.5 * x * (1.0 + scipy.special.erf(x / math.sqrt(2.0)))


UNARY = {
    "NEG": lambda a: -a,
    "ABS": np.abs,
    "EXP": np.exp,
    "LOG": np.log,
    "TANH": np.tanh,
    "ERF": scipy.special.erf,
    "SQRT": np.sqrt,
    "RSQRT": lambda a: 1.0 / np.sqrt(a),
    "RCP": lambda a: 1.0 / a,
    "SIGMOID": lambda a: 1.0 / (1.0 + np.exp(-a)),
    "GELU_TANH": _gelu_tanh,
    "GELU_ERF": _gelu_erf,
    "GELU_TANH_GRAD": _gelu_tanh_grad,
}


def _pow(a, b):
    """POW; an integer-valued scalar exponent is repeated multiplication (R11)."""
    if np.ndim(b) == 0 and float(b) == int(b) and 0 <= int(b) <= 8:
        n = int(b)
        r = np.ones_like(a)
        for _ in range(n):
            r = r * a
        return r
    return np.power(a, b)


BINARY = {
    "ADD": lambda a, b: a + b,
    "SUB": lambda a, b: a - b,
    "MUL": lambda a, b: a * b,
    "DIV": lambda a, b: a / b,
    "MAX": np.maximum,
    "MIN": np.minimum,
    "POW": _pow,
}

# ----------------------------------------------------------------------------
# Input widening (exact)
# ----------------------------------------------------------------------------


def widen(a: np.ndarray, dtype: str) -> np.ndarray:
    """Exact widening of the stored input bits to fp64.

    BF16 arrives as uint16 bit patterns: bf16 is the upper half of an IEEE
    binary32, so shifting left by 16 reconstructs the fp32 value exactly."""
    if dtype == "BF16":
        u = np.asarray(a, dtype=np.uint16).astype(np.uint32) << np.uint32(16)
        return u.view(np.float32).astype(np.float64)
    if dtype in ("F32", "F16"):
        return np.asarray(a).astype(np.float64)
    if dtype == "I32":
        return np.asarray(a, dtype=np.int64)
    raise ValueError(dtype)


# ----------------------------------------------------------------------------
# Graph analysis helpers
# ----------------------------------------------------------------------------


def _kinds(spec):
    """Kind of every named value (FULL / ROWVEC / COLVEC / SCALAR / LENGTHS)."""
    kind = {n: k for n, k, _ in spec["inputs"]}
    for op in spec["ops"]:
        name, typ = op[0], op[1]
        if typ == "const":
            kind[name] = "SCALAR"
        elif typ == "unary":
            kind[name] = kind[op[3]]
        elif typ == "binary":
            ka, kb = kind[op[3]], kind[op[4]]
            kind[name] = kb if ka == "SCALAR" else ka
        elif typ == "reduce":
            kind[name] = "ROWVEC" if op[3] == "ROW" else "COLVEC"
        elif typ == "broadcast":
            kind[name] = "FULL"
        else:
            raise ValueError(typ)
    return kind


def _operands(op):
    typ = op[1]
    if typ == "unary":
        return [op[3]]
    if typ == "binary":
        return [op[3], op[4]]
    if typ == "reduce":
        return [op[4]]
    if typ == "broadcast":
        return [op[3]]
    return []


def _levels(spec):
    """Number of column reductions on each value's dependency path: a column
    reduction is complete only after every row has been visited, so its
    consumers belong to the next pass over the rows."""
    level = {n: 0 for n, _, _ in spec["inputs"]}
    for op in spec["ops"]:
        lv = max([level[a] for a in _operands(op)] or [0])
        if op[1] == "reduce" and op[3] == "COL":
            lv += 1
        level[op[0]] = lv
    return level


# ----------------------------------------------------------------------------
# The evaluator
# ----------------------------------------------------------------------------


def evaluate_ragged(spec: dict, inputs: dict) -> dict:
    """Packed varlen layout (spec "segments", include/astitch.h
    astitch_graph_segments): segment s is an independent dense problem of
    rows_s x cols_s, read from the packed buffers through the segment table
    {row_start, cols, pitch, offset/8}.  Each segment is evaluated by
    :func:`evaluate` as the plain unmasked graph; FULL outputs are returned in
    the packed layout (1-D, pitch padding 0), ROWVEC outputs per global row."""
    seg = spec["segments"]
    table = np.asarray(inputs[seg["table"]], dtype=np.int64)
    R = int(spec["rows"])
    elems = int(seg["elems"])
    kind = _kinds(spec)
    assert not any(op[1] == "reduce" and op[3] == "COL" for op in spec["ops"]), \
        "packed varlen subgraphs are row-wise"
    outs = {}
    for n, _ in spec["outputs"]:
        outs[n] = np.zeros(elems if kind[n] == "FULL" else R, dtype=np.float64)
    sub_inputs_decl = [(n, k, d) for n, k, d in spec["inputs"] if k != "SEGMENTS"]
    for s in range(table.shape[0]):
        r0, cols, pitch, off = int(table[s, 0]), int(table[s, 1]), int(table[s, 2]), 8 * int(table[s, 3])
        r1 = int(table[s + 1, 0]) if s + 1 < table.shape[0] else R
        nr = r1 - r0
        if nr <= 0:
            continue
        sub = {"name": spec["name"], "rows": nr, "cols": cols, "inputs": sub_inputs_decl, "mask": None,
               "ops": spec["ops"], "outputs": spec["outputs"]}
        sin = {}
        for n, k, d in sub_inputs_decl:
            a = inputs[n]
            if k == "FULL":
                sin[n] = np.asarray(a)[off: off + nr * pitch].reshape(nr, pitch)[:, :cols]
            elif k == "ROWVEC":
                sin[n] = np.asarray(a)[r0:r1]
            elif k == "COLVEC":
                sin[n] = np.asarray(a)[:cols]
            else:
                raise ValueError(k)
        res = evaluate(sub, sin)
        for n, _ in spec["outputs"]:
            if kind[n] == "FULL":
                outs[n][off: off + nr * pitch].reshape(nr, pitch)[:, :cols] = res[n]
            else:
                outs[n][r0:r1] = res[n]
    return outs


def evaluate(spec: dict, inputs: dict, row_chunk: int = 16384) -> dict:
    """Evaluate ``spec`` on ``inputs`` (raw stored arrays keyed by input name).

    Returns ``{output name: fp64 ndarray}`` with shapes FULL [R,C], ROWVEC [R],
    COLVEC [C], SCALAR ().  Packed varlen specs go to :func:`evaluate_ragged`.
    """
    if spec.get("segments"):
        return evaluate_ragged(spec, inputs)
    R, C = int(spec["rows"]), int(spec["cols"])
    kind = _kinds(spec)
    level = _levels(spec)
    out_names = [n for n, _ in spec["outputs"]]
    mask = spec.get("mask")

    lengths = None
    if mask is not None:
        lengths = widen(inputs[mask["lengths"]], "I32")
        rps = int(mask["rows_per_segment"])

    # Whole-tensor values that do not depend on rows: COLVEC inputs, consts.
    glob = {}
    for n, k, d in spec["inputs"]:
        if k == "COLVEC":
            glob[n] = widen(inputs[n], d)
    for op in spec["ops"]:
        if op[1] == "const":
            glob[op[0]] = np.float64(op[2])

    def valid_for(r0, r1):
        if lengths is None:
            return None
        seg = np.arange(r0, r1) // rps
        return np.arange(C)[None, :] < lengths[seg][:, None]

    def eval_ops(env, valid, lvl):
        """Evaluate, in spec order on one row chunk, every op of level <= lvl.
        Column reductions of level-lvl operands produce chunk partials (combined
        by the caller); completed column reductions come from `glob`."""
        for op in spec["ops"]:
            name, typ = op[0], op[1]
            if typ == "const" or name in env:
                continue
            is_colred = typ == "reduce" and op[3] == "COL"
            if is_colred and level[op[4]] != lvl:
                continue  # complete (in glob) or not yet reachable
            if not is_colred and level[name] > lvl:
                continue
            if kind[name] == "COLVEC" and name in glob:
                env[name] = glob[name]
                continue
            if typ == "unary":
                env[name] = UNARY[op[2]](env[op[3]])
            elif typ == "binary":
                env[name] = BINARY[op[2]](env[op[3]], env[op[4]])
            elif typ == "broadcast":
                a = env[op[3]]
                nrows = env["__nrows__"]
                if op[2] == "ROW":
                    env[name] = np.broadcast_to(a[:, None], (nrows, C))
                else:
                    env[name] = np.broadcast_to(a[None, :], (nrows, C))
            elif typ == "reduce":
                a = env[op[4]]
                if op[3] == "ROW":
                    if op[2] == "SUM":
                        x = a if valid is None else np.where(valid, a, 0.0)
                        env[name] = np.add.reduce(x, axis=1)
                    else:
                        x = a if valid is None else np.where(valid, a, -np.inf)
                        env[name] = np.max(x, axis=1) if C > 0 else np.full(a.shape[0], -np.inf)
                else:
                    # column reduction: chunk partial, combined by the caller
                    if op[2] == "SUM":
                        x = a if valid is None else np.where(valid, a, 0.0)
                        env["__colpart__" + name] = np.add.reduce(x, axis=0)
                    else:
                        x = a if valid is None else np.where(valid, a, -np.inf)
                        env["__colpart__" + name] = (np.max(x, axis=0) if x.shape[0] > 0
                                                     else np.full(C, -np.inf))
            else:
                raise ValueError(typ)

    outs = {}
    for n in out_names:
        k = kind[n]
        shape = {"FULL": (R, C), "ROWVEC": (R,), "COLVEC": (C,), "SCALAR": ()}[k]
        outs[n] = np.zeros(shape, dtype=np.float64)

    colred = [op for op in spec["ops"] if op[1] == "reduce" and op[3] == "COL"]
    colacc = {}
    for op in colred:
        colacc[op[0]] = np.zeros(C) if op[2] == "SUM" else np.full(C, -np.inf)

    def chunk_env(r0, r1):
        env = dict(glob)
        env["__nrows__"] = r1 - r0
        for n, k, d in spec["inputs"]:
            if k == "FULL":
                env[n] = widen(inputs[n][r0:r1], d)
            elif k == "ROWVEC":
                env[n] = widen(inputs[n][r0:r1], d)
        return env

    def store(env, r0, r1, valid, names):
        for n in names:
            if n not in env:
                continue
            k = kind[n]
            if k == "FULL":
                v = np.asarray(env[n], dtype=np.float64)
                if valid is not None:
                    v = np.where(valid, v, 0.0)
                outs[n][r0:r1] = v
            elif k == "ROWVEC":
                outs[n][r0:r1] = env[n]
            elif k == "COLVEC":
                outs[n][:] = env[n]

    D = max(level.values()) if level else 0
    with np.errstate(all="ignore"):
        # one pass over the rows per level of dependent column reductions
        for lvl in range(D + 1):
            red_here = [op for op in colred if level[op[4]] == lvl]
            rows_out = [n for n in out_names if level[n] == lvl and kind[n] in ("FULL", "ROWVEC")]
            if lvl == 0 or red_here or rows_out:
                for r0 in range(0, R, row_chunk):
                    r1 = min(R, r0 + row_chunk)
                    valid = valid_for(r0, r1)
                    env = chunk_env(r0, r1)
                    eval_ops(env, valid, lvl)
                    for op in red_here:
                        p = env["__colpart__" + op[0]]
                        if op[2] == "SUM":
                            colacc[op[0]] = colacc[op[0]] + p
                        else:
                            colacc[op[0]] = np.maximum(colacc[op[0]], p)
                    store(env, r0, r1, valid, [n for n in out_names if level[n] == lvl])
            # these column reductions are complete: their COLVEC consumers
            for op in red_here:
                glob[op[0]] = colacc[op[0]]
            for op in spec["ops"]:
                name, typ = op[0], op[1]
                if kind[name] != "COLVEC" or name in glob or level[name] > lvl + 1:
                    continue
                if typ == "reduce":
                    continue  # a later level's column reduction
                if typ == "unary":
                    glob[name] = UNARY[op[2]](glob[op[3]])
                elif typ == "binary":
                    glob[name] = BINARY[op[2]](glob[op[3]], glob[op[4]])
        for n in out_names:
            if kind[n] == "COLVEC" and n in glob:
                outs[n][:] = glob[n]
            elif kind[n] == "SCALAR":
                outs[n] = np.float64(glob[n])
    return outs


def evaluate_columns(spec: dict, inputs: dict, cols: np.ndarray, row_chunk: int = 65536) -> dict:
    """Evaluate a spec whose ops never mix columns (no ROW reduce, no ROWVEC,
    no mask) on a subset of columns: the sub-problem is the same graph on
    ``inputs[..., cols]``.  Used for sampled parity at full size (e.g. C5's
    column sums over all 1,048,576 rows for a few columns)."""
    kind = _kinds(spec)
    assert spec.get("mask") is None
    for op in spec["ops"]:
        assert not (op[1] == "reduce" and op[3] == "ROW"), "row reduce mixes columns"
        assert not (op[1] == "broadcast" and op[2] == "ROW"), "row broadcast mixes columns"
    assert all(k != "ROWVEC" for k in kind.values())
    sub = dict(spec)
    sub["cols"] = int(len(cols))
    sub_inputs = {}
    for n, k, d in spec["inputs"]:
        if k == "FULL":
            sub_inputs[n] = np.ascontiguousarray(inputs[n][:, cols])
        elif k == "COLVEC":
            sub_inputs[n] = np.ascontiguousarray(inputs[n][cols])
        else:
            sub_inputs[n] = inputs[n]
    return evaluate(sub, sub_inputs, row_chunk=row_chunk)


def evaluate_rows(spec: dict, inputs: dict, rows: np.ndarray) -> dict:
    """Evaluate the FULL/ROWVEC outputs of a spec with no column reduction on a
    subset of rows (rows are independent units there): the sub-problem is the
    same graph on the selected rows, with the mask lengths re-indexed."""
    kind = _kinds(spec)
    assert not any(op[1] == "reduce" and op[3] == "COL" for op in spec["ops"])
    rows = np.asarray(rows, dtype=np.int64)
    sub = dict(spec)
    sub["rows"] = int(len(rows))
    sub_inputs = {}
    mask = spec.get("mask")
    for n, k, d in spec["inputs"]:
        if k in ("FULL", "ROWVEC"):
            sub_inputs[n] = np.ascontiguousarray(inputs[n][rows])
        else:
            sub_inputs[n] = inputs[n]
    if mask is not None:
        L = np.asarray(inputs[mask["lengths"]])
        sub_inputs[mask["lengths"]] = L[rows // int(mask["rows_per_segment"])].astype(np.int32)
        sub["mask"] = {"lengths": mask["lengths"], "rows_per_segment": 1}
    del kind
    return evaluate(sub, sub_inputs)
