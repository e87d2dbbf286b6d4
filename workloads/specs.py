"""Declarative subgraph specs for the benchmark and pin workloads (DATA ONLY).

This module holds no arithmetic of the method: each spec is a plain list of
tuples naming the ops of a memory-intensive subgraph, in topological order.
Both sides read it independently:

* the product binding (``paper_conf_asplos_zhengyzlzzzlyzs22_b200.Graph.from_spec``)
  replays it through the C-ABI graph builder (``include/astitch.h``);
* the oracle (``oracle/evaluator.py``) has its own reader and evaluates the ops
  one by one in fp64.

Spec format (all strings upper-case as in the C-ABI enums)::

    {
      "name": str, "rows": int, "cols": int,
      "inputs":  [(name, kind, dtype), ...]        kind in FULL|ROWVEC|COLVEC|LENGTHS|SEGMENTS
      "mask":    None | {"lengths": name, "rows_per_segment": int}
      "segments": (packed varlen only) {"table": name, "batches", "heads", "min_len"}
                 -> workloads.gen.ragged_spec adds "seg_rows", "seg_cols", "elems"
      "ops":     [(name, "const", value)
                  (name, "unary", UNOP, a)
                  (name, "binary", BINOP, a, b)
                  (name, "reduce", SUM|RMAX, ROW|COL, a)
                  (name, "broadcast", ROW|COL, a)], ...
      "outputs": [(name, dtype), ...]
    }

The op vocabulary follows the paper's taxonomy (Sec. 2.1):
element-wise (light / heavy), broadcast, row-reduce and column-reduce.
The five configs C1..C5 are BASELINE.json ``configs[0..4]``; the readings used
to make each one concrete are SURVEY.md Sec. 8(c) (listed again in DESIGN.md).
"""

from __future__ import annotations

import copy

# ---------------------------------------------------------------------------
# C1: softmax fp32 [32,128]  (BASELINE.json configs[0]; reduce_max, sub, exp,
# reduce_sum, div as one regional-stitched kernel)
# ---------------------------------------------------------------------------
C1_SOFTMAX = {
    "name": "C1_softmax_f32",
    "rows": 32,
    "cols": 128,
    "inputs": [("x", "FULL", "F32")],
    "mask": None,
    "ops": [
        ("m", "reduce", "RMAX", "ROW", "x"),
        ("mb", "broadcast", "ROW", "m"),
        ("xm", "binary", "SUB", "x", "mb"),
        ("e", "unary", "EXP", "xm"),
        ("s", "reduce", "SUM", "ROW", "e"),
        ("sb", "broadcast", "ROW", "s"),
        ("y", "binary", "DIV", "e", "sb"),
    ],
    "outputs": [("y", "F32")],
}

# ---------------------------------------------------------------------------
# C2: BERT-base bias + residual + LayerNorm + GELU, bf16 [4096,768]
# (configs[1]; batch 32 x seq 128 = 4096 rows, hidden 768). Readings R5, R7:
# gelu = tanh form, biased variance, eps = 1e-12 inside the sqrt.
# ---------------------------------------------------------------------------
C2_BERT_LN_GELU = {
    "name": "C2_bert_bias_residual_layernorm_gelu_bf16",
    "rows": 4096,
    "cols": 768,
    "inputs": [
        ("x", "FULL", "BF16"),
        ("r", "FULL", "BF16"),
        ("b", "COLVEC", "BF16"),
        ("gamma", "COLVEC", "BF16"),
        ("beta", "COLVEC", "BF16"),
    ],
    "mask": None,
    "ops": [
        ("bb", "broadcast", "COL", "b"),
        ("xb", "binary", "ADD", "x", "bb"),
        ("h", "binary", "ADD", "xb", "r"),
        ("hs", "reduce", "SUM", "ROW", "h"),
        ("ncols", "const", 768.0),
        ("mu", "binary", "DIV", "hs", "ncols"),
        ("mub", "broadcast", "ROW", "mu"),
        ("c", "binary", "SUB", "h", "mub"),
        ("c2", "binary", "MUL", "c", "c"),
        ("vs", "reduce", "SUM", "ROW", "c2"),
        ("var", "binary", "DIV", "vs", "ncols"),
        ("eps", "const", 1e-12),
        ("ve", "binary", "ADD", "var", "eps"),
        ("rstd", "unary", "RSQRT", "ve"),
        ("rstdb", "broadcast", "ROW", "rstd"),
        ("xhat", "binary", "MUL", "c", "rstdb"),
        ("gb", "broadcast", "COL", "gamma"),
        ("yg", "binary", "MUL", "xhat", "gb"),
        ("betab", "broadcast", "COL", "beta"),
        ("y", "binary", "ADD", "yg", "betab"),
        ("o", "unary", "GELU_TANH", "y"),
    ],
    "outputs": [("o", "BF16")],
}

# ---------------------------------------------------------------------------
# C3: Transformer attention softmax bf16 [64*16*512, 512] with irregular key
# lengths 37..512 (configs[2]).  Reading R9: key-padding mask, one length per
# batch of 16 heads x 512 query rows = 8192 rows per segment.
# ---------------------------------------------------------------------------
C3_ATTN_SOFTMAX = {
    "name": "C3_attention_masked_softmax_bf16",
    "rows": 64 * 16 * 512,
    "cols": 512,
    "inputs": [("s", "FULL", "BF16"), ("L", "LENGTHS", "I32")],
    "mask": {"lengths": "L", "rows_per_segment": 16 * 512},
    "ops": [
        ("scale", "const", 0.125),
        ("a", "binary", "MUL", "s", "scale"),
        ("m", "reduce", "RMAX", "ROW", "a"),
        ("mb", "broadcast", "ROW", "m"),
        ("am", "binary", "SUB", "a", "mb"),
        ("e", "unary", "EXP", "am"),
        ("z", "reduce", "SUM", "ROW", "e"),
        ("zb", "broadcast", "ROW", "z"),
        ("p", "binary", "DIV", "e", "zb"),
    ],
    "outputs": [("p", "BF16")],
}

# C3v: the same attention softmax on the PACKED varlen layout (SURVEY 8(f)
# f2(ii); the paper's irregular shapes): batch b contributes
# heads x L_b query rows of L_b keys each, stored back to back with no padding
# (row pitch = L_b rounded up to 8 elements).  `rows` / the segment lists are
# filled in by workloads.gen.ragged_spec from the seeded lengths (the same
# draw as C3's L); cols = the maximum row length.
C3V_ATTN_SOFTMAX_VARLEN = {
    "name": "C3v_attention_softmax_varlen_bf16",
    "rows": None,
    "cols": 512,
    "inputs": [("s", "FULL", "BF16"), ("S", "SEGMENTS", "I32")],
    "mask": None,
    "segments": {"table": "S", "batches": 64, "heads": 16, "min_len": 37},
    "ops": [op for op in C3_ATTN_SOFTMAX["ops"]],
    "outputs": [("p", "BF16")],
}

# ---------------------------------------------------------------------------
# C4: DIEN-style many tiny rows, reduce+broadcast chains fp32 [2,000,000, 36]
# (configs[3]).  Row standardisation; eps = 1e-5 (reading R7).
# ---------------------------------------------------------------------------
C4_DIEN_ROWNORM = {
    "name": "C4_dien_row_standardise_f32",
    "rows": 2_000_000,
    "cols": 36,
    "inputs": [("x", "FULL", "F32")],
    "mask": None,
    "ops": [
        ("xs", "reduce", "SUM", "ROW", "x"),
        ("ncols", "const", 36.0),
        ("mu", "binary", "DIV", "xs", "ncols"),
        ("mub", "broadcast", "ROW", "mu"),
        ("c", "binary", "SUB", "x", "mub"),
        ("c2", "binary", "MUL", "c", "c"),
        ("vs", "reduce", "SUM", "ROW", "c2"),
        ("var", "binary", "DIV", "vs", "ncols"),
        ("eps", "const", 1e-5),
        ("ve", "binary", "ADD", "var", "eps"),
        ("rstd", "unary", "RSQRT", "ve"),
        ("rstdb", "broadcast", "ROW", "rstd"),
        ("o", "binary", "MUL", "c", "rstdb"),
    ],
    "outputs": [("o", "F32")],
}

# ---------------------------------------------------------------------------
# C5: training bias-gradient: dz = dy * gelu_tanh'(z); db = col_sum(dz);
# b_new = b - 2^-7 * db (configs[4]; readings R3, R4, R10).  Global stitching:
# the column reduce feeds a consumer after the grid barrier.
# ---------------------------------------------------------------------------
C5_BIAS_GRAD = {
    "name": "C5_bias_gelu_backward_colreduce_bf16",
    "rows": 1_048_576,
    "cols": 1024,
    "inputs": [("dy", "FULL", "BF16"), ("z", "FULL", "BF16"), ("b", "COLVEC", "F32")],
    "mask": None,
    "ops": [
        ("g", "unary", "GELU_TANH_GRAD", "z"),
        ("dz", "binary", "MUL", "dy", "g"),
        ("db", "reduce", "SUM", "COL", "dz"),
        ("lr", "const", 0.0078125),
        ("step", "binary", "MUL", "db", "lr"),
        ("b_new", "binary", "SUB", "b", "step"),
    ],
    "outputs": [("dz", "BF16"), ("db", "F32"), ("b_new", "F32")],
}

# Exactness variant of C5 (SURVEY Sec. 8(c) pins): small-integer operands make
# every product and every fp32 column partial exact, so db must match bitwise.
C5_INT_EXACT = {
    "name": "C5int_colreduce_exact_bf16",
    "rows": 1_048_576,
    "cols": 1024,
    "inputs": [("dy", "FULL", "BF16"), ("z", "FULL", "BF16"), ("b", "COLVEC", "F32")],
    "mask": None,
    "ops": [
        ("dz", "binary", "MUL", "dy", "z"),
        ("db", "reduce", "SUM", "COL", "dz"),
        ("lr", "const", 0.0078125),
        ("step", "binary", "MUL", "db", "lr"),
        ("b_new", "binary", "SUB", "b", "step"),
    ],
    "outputs": [("dz", "BF16"), ("db", "F32"), ("b_new", "F32")],
}

# ---------------------------------------------------------------------------
# Fig. 5: power<2> -> broadcast<2,128> -> add<2,128>.  The heavy
# element-wise producer lives on the [2] row vector and must be computed once
# per row, not once per consumer element.
# ---------------------------------------------------------------------------
FIG5_POWER_BCAST_ADD = {
    "name": "fig5_power_broadcast_add",
    "rows": 2,
    "cols": 128,
    "inputs": [("p", "ROWVEC", "F32"), ("y", "FULL", "F32")],
    "mask": None,
    "ops": [
        ("three", "const", 3.0),
        ("pw", "binary", "POW", "p", "three"),
        ("pwb", "broadcast", "ROW", "pw"),
        ("o", "binary", "ADD", "y", "pwb"),
    ],
    "outputs": [("o", "F32")],
}

# ---------------------------------------------------------------------------
# Fig. 7(a) / Fig. 9, topology reading of SURVEY
# Sec. 4 (partially unpinned: the figure is lost).  reduce.1 regional,
# power.1 / reduce.2 global, multiply.1 the stitch output.
# ---------------------------------------------------------------------------
FIG7A_MIXED = {
    "name": "fig7a_regional_global_mixed",
    "rows": 300,
    "cols": 96,
    "inputs": [("x", "FULL", "F32"), ("p2", "ROWVEC", "F32")],
    "mask": None,
    "ops": [
        ("reduce1", "reduce", "SUM", "ROW", "x"),
        ("divide1", "binary", "DIV", "reduce1", "p2"),
        ("broadcast1", "broadcast", "ROW", "divide1"),
        ("add1", "binary", "SUB", "x", "broadcast1"),
        ("two", "const", 2.0),
        ("power1", "binary", "POW", "add1", "two"),
        ("reduce2", "reduce", "SUM", "COL", "power1"),
        ("broadcast2", "broadcast", "COL", "reduce2"),
        # multiply.1 consumes power.1 across the barrier, which is what makes
        # power.1 "global" in P:L198 (its value is buffered in HBM)
        ("multiply1", "binary", "MUL", "power1", "broadcast2"),
    ],
    "outputs": [("multiply1", "F32")],
}

# Fig. 6: the two poor-parallelism row-reduce shapes.
FIG6A_MANY_SHORT_ROWS = {
    "name": "fig6a_rowsum_750000x32",
    "rows": 750_000,
    "cols": 32,
    "inputs": [("x", "FULL", "F32")],
    "mask": None,
    "ops": [("s", "reduce", "SUM", "ROW", "x")],
    "outputs": [("s", "F32")],
}

FIG6B_FEW_LONG_ROWS = {
    "name": "fig6b_rowsum_64x30000",
    "rows": 64,
    "cols": 30_000,
    "inputs": [("x", "FULL", "F32")],
    "mask": None,
    "ops": [("s", "reduce", "SUM", "ROW", "x")],
    "outputs": [("s", "F32")],
}

# Training BatchNorm forward (the BN of CRNN-style convnets, Table 2):
# two DEPENDENT column reductions (mean, then variance of the centred values),
# i.e. two grid barriers in one stitched kernel.  rows = N*H*W, cols = channels.
# The const named "nrows" follows the row count (see resized()).
BN_TRAIN_FWD = {
    "name": "batchnorm_train_forward_f32",
    "rows": 32 * 28 * 28,
    "cols": 128,
    "inputs": [("x", "FULL", "F32"), ("gamma", "COLVEC", "F32"), ("beta", "COLVEC", "F32")],
    "mask": None,
    "ops": [
        ("s1", "reduce", "SUM", "COL", "x"),
        ("nrows", "const", float(32 * 28 * 28)),
        ("mean", "binary", "DIV", "s1", "nrows"),
        ("meanb", "broadcast", "COL", "mean"),
        ("xc", "binary", "SUB", "x", "meanb"),
        ("xc2", "binary", "MUL", "xc", "xc"),
        ("s2", "reduce", "SUM", "COL", "xc2"),
        ("var", "binary", "DIV", "s2", "nrows"),
        ("eps", "const", 1e-5),
        ("ve", "binary", "ADD", "var", "eps"),
        ("rstd", "unary", "RSQRT", "ve"),
        ("rstdb", "broadcast", "COL", "rstd"),
        ("xhat", "binary", "MUL", "xc", "rstdb"),
        ("gb", "broadcast", "COL", "gamma"),
        ("yg", "binary", "MUL", "xhat", "gb"),
        ("bb", "broadcast", "COL", "beta"),
        ("y", "binary", "ADD", "yg", "bb"),
    ],
    "outputs": [("y", "F32"), ("mean", "F32"), ("var", "F32")],
}

# LM-head softmax over a 128K vocabulary, bf16 [4096 tokens, 128256]: rows of
# 256 KB, longer than any team's registers -> the row_stream template (one
# pass per row-reduction level: max | sum | normalise).
LM_SOFTMAX = {
    "name": "lm_head_softmax_bf16_4096x128256",
    "rows": 4096,
    "cols": 128256,
    "inputs": [("x", "FULL", "BF16")],
    "mask": None,
    "ops": [op for op in C1_SOFTMAX["ops"]],
    "outputs": [("y", "BF16")],
}

# Remote stitching: two subgraphs with no data dependency merged into
# one stitch op (the "independent" scheme between them), one kernel.
REMOTE_TWO_SUBGRAPHS = {
    "name": "remote_softmax_and_rowsum",
    "rows": 3000,
    "cols": 256,
    "inputs": [("x", "FULL", "BF16"), ("y", "FULL", "F32")],
    "mask": None,
    "ops": [
        ("m", "reduce", "RMAX", "ROW", "x"),
        ("mb", "broadcast", "ROW", "m"),
        ("xm", "binary", "SUB", "x", "mb"),
        ("e", "unary", "EXP", "xm"),
        ("s", "reduce", "SUM", "ROW", "e"),
        ("sb", "broadcast", "ROW", "s"),
        ("p", "binary", "DIV", "e", "sb"),
        ("ys", "reduce", "SUM", "ROW", "y"),
        ("ya", "unary", "ABS", "y"),
        ("yn", "reduce", "RMAX", "ROW", "ya"),
    ],
    "outputs": [("p", "BF16"), ("ys", "F32"), ("yn", "F32")],
}

CONFIGS = {
    "C1": C1_SOFTMAX,
    "C2": C2_BERT_LN_GELU,
    "C3": C3_ATTN_SOFTMAX,
    "C4": C4_DIEN_ROWNORM,
    "C5": C5_BIAS_GRAD,
}

EXTRA = {
    "C3v": C3V_ATTN_SOFTMAX_VARLEN,
    "C5int": C5_INT_EXACT,
    "fig5": FIG5_POWER_BCAST_ADD,
    "fig7a": FIG7A_MIXED,
    "fig6a": FIG6A_MANY_SHORT_ROWS,
    "fig6b": FIG6B_FEW_LONG_ROWS,
    "remote": REMOTE_TWO_SUBGRAPHS,
    "bn": BN_TRAIN_FWD,
    "lmsoftmax": LM_SOFTMAX,
}

ALL = {**CONFIGS, **EXTRA}


def get(name: str, rows: int | None = None, cols: int | None = None) -> dict:
    """Return a deep copy of spec ``name`` with optional shape overrides."""
    return resized(ALL[name], rows, cols)


def resized(spec: dict, rows: int | None = None, cols: int | None = None) -> dict:
    """Copy of ``spec`` at another shape.  A const op named ``ncols`` (the mean
    divisor of the LayerNorm-style specs) follows the new column count, one
    named ``nrows`` (BatchNorm) the new row count."""
    s = copy.deepcopy(spec)
    if rows is not None:
        s["rows"] = int(rows)
        s["ops"] = [(o[0], "const", float(rows)) if (o[1] == "const" and o[0] == "nrows") else o
                    for o in s["ops"]]
    if cols is not None:
        s["cols"] = int(cols)
        s["ops"] = [(o[0], "const", float(cols)) if (o[1] == "const" and o[0] == "ncols") else o
                    for o in s["ops"]]
    return s
