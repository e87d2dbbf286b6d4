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
second pass once every chunk has been reduced.  This is the definition,
split over rows; it has no blocking across columns and no fusion.
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


def _after_colreduce(spec):
    """Values that depend (transitively) on a column reduction."""
    post = set()
    for op in spec["ops"]:
        name, typ = op[0], op[1]
        if typ == "reduce" and op[3] == "COL":
            post.add(name)
        elif typ in ("unary", "broadcast") and op[-1] in post:
            post.add(name)
        elif typ == "binary" and (op[3] in post or op[4] in post):
            post.add(name)
        elif typ == "reduce" and op[4] in post:
            if op[3] == "COL":
                raise NotImplementedError("a column reduction downstream of another one")
            post.add(name)
    return post


# ----------------------------------------------------------------------------
# The evaluator
# ----------------------------------------------------------------------------


def evaluate(spec: dict, inputs: dict, row_chunk: int = 16384) -> dict:
    """Evaluate ``spec`` on ``inputs`` (raw stored arrays keyed by input name).

    Returns ``{output name: fp64 ndarray}`` with shapes FULL [R,C], ROWVEC [R],
    COLVEC [C], SCALAR ().
    """
    R, C = int(spec["rows"]), int(spec["cols"])
    kind = _kinds(spec)
    post = _after_colreduce(spec)
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

    def eval_ops(env, valid, second_pass):
        """Evaluate the ops in order on one row chunk.  First pass: only the
        ops that do not depend on a column reduction.  Second pass: the rest."""
        for op in spec["ops"]:
            name, typ = op[0], op[1]
            if typ == "const":
                continue
            if name in env and not (second_pass and name in post):
                continue
            is_colred = typ == "reduce" and op[3] == "COL"
            if not second_pass and name in post and not is_colred:
                continue
            if second_pass and is_colred:
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

    with np.errstate(all="ignore"):
        # pass 1: everything not downstream of a column reduction
        for r0 in range(0, R, row_chunk):
            r1 = min(R, r0 + row_chunk)
            valid = valid_for(r0, r1)
            env = chunk_env(r0, r1)
            eval_ops(env, valid, second_pass=False)
            for op in colred:
                p = env.get("__colpart__" + op[0])
                if p is None:
                    continue
                if op[2] == "SUM":
                    colacc[op[0]] = colacc[op[0]] + p
                else:
                    colacc[op[0]] = np.maximum(colacc[op[0]], p)
            store(env, r0, r1, valid, [n for n in out_names if n not in post])

        if colred:
            # the column reductions are complete: evaluate their COLVEC consumers
            for k_, v in colacc.items():
                glob[k_] = v
            cenv = dict(glob)
            cenv["__nrows__"] = 0
            for op in spec["ops"]:
                name, typ = op[0], op[1]
                if name not in post or kind[name] != "COLVEC" or name in glob:
                    continue
                if typ == "unary":
                    glob[name] = UNARY[op[2]](cenv[op[3]])
                elif typ == "binary":
                    glob[name] = BINARY[op[2]](cenv[op[3]], cenv[op[4]])
                cenv[name] = glob[name]
            for n in out_names:
                if kind[n] == "COLVEC":
                    outs[n][:] = glob[n]
                elif kind[n] == "SCALAR":
                    outs[n] = np.float64(glob[n])

            # pass 2: FULL / ROWVEC values downstream of a column reduction
            need2 = [n for n in out_names if n in post and kind[n] in ("FULL", "ROWVEC")]
            if need2:
                for r0 in range(0, R, row_chunk):
                    r1 = min(R, r0 + row_chunk)
                    valid = valid_for(r0, r1)
                    env = chunk_env(r0, r1)
                    eval_ops(env, valid, second_pass=False)
                    env.update({k_: glob[k_] for k_ in glob})
                    eval_ops(env, valid, second_pass=True)
                    store(env, r0, r1, valid, need2)
        else:
            for n in out_names:
                if kind[n] == "COLVEC" and n in glob:
                    outs[n][:] = glob[n]
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
