"""Pins for the fp64 oracle (CPU only, -m "not gpu").

Each test checks oracle/evaluator.py against something other than itself:
values the paper prints (tests/golden/, with citations), closed forms,
invariants, textbook special cases, brute force on tiny inputs.  Together they
are chosen so that a dropped term, a wrong sign or index, or a transposed
operand in the oracle fails at least one of them.
"""

import math
import os

import numpy as np
import pytest
import scipy.stats

from oracle import evaluate, evaluate_columns, evaluate_rows, widen
from oracle.evaluator import UNARY
from workloads import gen, specs

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def golden(name):
    d = {}
    with open(os.path.join(GOLD, name)) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            k, v = line.split(":", 1)
            d[k.strip()] = [float(t) for t in v.split()]
    return d


def spec_tiny(ops, inputs, outputs, rows, cols, mask=None):
    return {"name": "tiny", "rows": rows, "cols": cols, "inputs": inputs, "mask": mask,
            "ops": ops, "outputs": outputs}


# ---------------------------------------------------------------- reductions

def test_fig3_reduce_golden():
    g = golden("fig3_reduce.txt")
    s = spec_tiny([("s", "reduce", "SUM", "ROW", "x")], [("x", "FULL", "F32")],
                  [("s", "F32")], 1, 3)
    out = evaluate(s, {"x": np.array([g["row"]], dtype=np.float32)})
    assert out["s"][0] == g["sum"][0]


@pytest.mark.parametrize("redop", ["SUM", "RMAX"])
@pytest.mark.parametrize("axis", ["ROW", "COL"])
@pytest.mark.parametrize("masked", [False, True])
def test_reduce_bruteforce(redop, axis, masked):
    rng = np.random.default_rng(11)
    R, C, rps = 7, 5, 2
    x = rng.standard_normal((R, C)).astype(np.float32)
    L = np.array([5, 0, 3, 1], dtype=np.int32)
    inputs = [("x", "FULL", "F32")]
    mask = None
    if masked:
        inputs.append(("L", "LENGTHS", "I32"))
        mask = {"lengths": "L", "rows_per_segment": rps}
    s = spec_tiny([("r", "reduce", redop, axis, "x")], inputs, [("r", "F32")], R, C, mask)
    out = evaluate(s, {"x": x, "L": L})["r"]

    def ok(r, c):
        return (not masked) or c < L[r // rps]

    ident = 0.0 if redop == "SUM" else -math.inf
    if axis == "ROW":
        for r in range(R):
            acc = ident
            for c in range(C):
                if ok(r, c):
                    acc = acc + float(x[r, c]) if redop == "SUM" else max(acc, float(x[r, c]))
            assert out[r] == pytest.approx(acc, abs=1e-12) or (acc == -math.inf and out[r] == -math.inf)
    else:
        for c in range(C):
            acc = ident
            for r in range(R):
                if ok(r, c):
                    acc = acc + float(x[r, c]) if redop == "SUM" else max(acc, float(x[r, c]))
            assert out[c] == pytest.approx(acc, abs=1e-12) or (acc == -math.inf and out[c] == -math.inf)


def test_colsum_exact_small_integers_c5int():
    spec = specs.get("C5int", rows=3 * gen.CHUNK_ROWS + 77, cols=64)
    x = gen.generate("C5int", spec)
    out = evaluate(spec, x, row_chunk=5000)
    dy = widen(x["dy"], "BF16").astype(np.int64)
    z = widen(x["z"], "BF16").astype(np.int64)
    exact = (dy * z).sum(axis=0)                       # integer arithmetic, exact
    assert np.array_equal(out["db"], exact.astype(np.float64))
    assert np.array_equal(out["dz"], (dy * z).astype(np.float64))


def test_colsum_row_permutation_invariance():
    spec = specs.get("C5", rows=1000, cols=32)
    x = gen.generate("C5", spec)
    perm = np.random.default_rng(0).permutation(1000)
    xp = dict(x, dy=x["dy"][perm], z=x["z"][perm])
    a = evaluate(spec, x, row_chunk=128)["db"]
    b = evaluate(spec, xp, row_chunk=333)["db"]
    np.testing.assert_allclose(a, b, rtol=1e-13, atol=1e-12)


def test_bias_step_golden():
    g = golden("bias_step.txt")
    spec = specs.get("C5int", rows=3, cols=1)
    dz = np.array(g["dz_col"], dtype=np.float32)
    x = {"dy": gen.f32_to_bf16_bits(dz[:, None]), "z": gen.f32_to_bf16_bits(np.ones((3, 1), np.float32)),
         "b": np.array(g["b"], dtype=np.float32)}
    out = evaluate(spec, x)
    assert out["db"][0] == g["db"][0]
    assert out["b_new"][0] == g["b_new"][0]


# ---------------------------------------------------------------- softmax

def test_softmax_rows_sum_to_one_c1():
    spec = specs.get("C1")
    x = gen.generate("C1", spec)
    y = evaluate(spec, x)["y"]
    np.testing.assert_allclose(y.sum(axis=1), 1.0, rtol=0, atol=1e-14)
    assert (y > 0).all()
    # shift invariance: adding a per-row constant leaves softmax unchanged
    xs = {"x": (x["x"] + np.float32(3.0)).astype(np.float32)}
    ys = evaluate(spec, xs)["y"]
    ref = evaluate(spec, {"x": x["x"]})["y"]
    # the shifted fp32 input is rounded, so compare against softmax of the rounded input
    xd = xs["x"].astype(np.float64)
    e = np.exp(xd - xd.max(axis=1, keepdims=True))
    np.testing.assert_allclose(ys, e / e.sum(axis=1, keepdims=True), rtol=1e-13)
    del ref


def test_softmax_closed_forms():
    g = golden("softmax_closed_form.txt")
    n = int(g["n"][0])
    spec = specs.get("C1", rows=2, cols=n)
    x = np.stack([np.arange(n, dtype=np.float32), np.full(n, 0.7, np.float32)])
    y = evaluate(spec, {"x": x})["y"]
    assert y[0, n - 1] == pytest.approx(g["last"][0], rel=1e-14)
    np.testing.assert_allclose(y[0, :-1] / y[0, 1:], math.exp(-1), rtol=1e-13)
    np.testing.assert_allclose(y[1], 1.0 / n, rtol=1e-15)            # constant row -> 1/C


def test_masked_softmax_golden_and_tail():
    g = golden("softmax_closed_form.txt")
    spec = specs.get("C3", rows=3, cols=4)
    spec["mask"]["rows_per_segment"] = 1
    row = np.array(g["masked_row"], dtype=np.float64)
    # C3 scales by 0.125: feed 8*row so the scaled logits are exactly `row`
    s = gen.f32_to_bf16_bits(np.stack([8 * row, 8 * row, 8 * row]).astype(np.float32))
    a = widen(s, "BF16") * 0.125
    L = np.array([int(g["masked_L"][0]), 0, 4], dtype=np.int32)
    p = evaluate(spec, {"s": s, "L": L})["p"]
    # row 0: bf16 rounding moves ln2*8 slightly; compare to the exact softmax of the stored bits
    e = np.exp(a[0, :2] - a[0, :2].max())
    np.testing.assert_allclose(p[0, :2], e / e.sum(), rtol=1e-14)
    np.testing.assert_allclose(p[0], g["masked_out"], atol=3e-3)   # golden up to bf16 input rounding
    assert (p[0, 2:] == 0).all()
    assert (p[1] == 0).all()                                       # fully masked row (R14)
    assert p[2].sum() == pytest.approx(1.0, abs=1e-14)


def test_c3_masked_rows_sum_and_zero_tail():
    spec = specs.get("C3", rows=3 * 64, cols=512)
    spec["mask"]["rows_per_segment"] = 64
    x = gen.generate("C3", spec)
    p = evaluate(spec, x)["p"]
    L = x["L"]
    for r in range(spec["rows"]):
        l_ = L[r // 64]
        assert p[r, :l_].sum() == pytest.approx(1.0, abs=1e-13)
        assert (p[r, l_:] == 0).all()


# ---------------------------------------------------------------- layernorm

def test_layernorm_golden_1234():
    g = golden("layernorm_1234.txt")
    spec = specs.get("C4", rows=1, cols=4)
    o = evaluate(spec, {"x": np.array([g["x"]], dtype=np.float32)})["o"]
    np.testing.assert_allclose(o[0], g["o"], rtol=1e-14)


def test_layernorm_invariants_c4():
    spec = specs.get("C4", rows=500)
    x = gen.generate("C4", spec)
    o = evaluate(spec, x)["o"]
    xd = x["x"].astype(np.float64)
    v = xd.var(axis=1)
    np.testing.assert_allclose(o.mean(axis=1), 0.0, atol=1e-14)
    np.testing.assert_allclose(o.var(axis=1), v / (v + 1e-5), rtol=1e-12)


def test_layernorm_invariants_c2_before_affine():
    spec = specs.get("C2", rows=64)
    spec["outputs"] = [("xhat", "F32"), ("y", "F32"), ("o", "BF16"), ("h", "F32")]
    x = gen.generate("C2", spec)
    out = evaluate(spec, x)
    h = out["h"]
    np.testing.assert_allclose(
        h, widen(x["x"], "BF16") + widen(x["b"], "BF16")[None, :] + widen(x["r"], "BF16"), rtol=1e-15)
    v = h.var(axis=1)
    np.testing.assert_allclose(out["xhat"].mean(axis=1), 0.0, atol=1e-14)
    np.testing.assert_allclose(out["xhat"].var(axis=1), v / (v + 1e-12), rtol=1e-12)
    # affine with gamma, beta applied per column, then GELU
    gm, bt = widen(x["gamma"], "BF16"), widen(x["beta"], "BF16")
    np.testing.assert_allclose(out["y"], out["xhat"] * gm[None, :] + bt[None, :], rtol=1e-14, atol=1e-15)
    np.testing.assert_allclose(out["o"], UNARY["GELU_TANH"](out["y"]), rtol=1e-15)


# ---------------------------------------------------------------- GELU

def test_gelu_values_and_identities():
    g = golden("gelu_values.txt")
    one = np.array([1.0])
    assert UNARY["GELU_ERF"](one)[0] == pytest.approx(g["gelu_erf_1"][0], rel=1e-15)
    assert UNARY["GELU_TANH"](one)[0] == pytest.approx(g["gelu_tanh_1"][0], rel=1e-15)
    x = np.linspace(-6, 6, 2001)
    for f in ("GELU_TANH", "GELU_ERF"):
        np.testing.assert_allclose(UNARY[f](x) - UNARY[f](-x), x, atol=1e-14)   # odd part = x/2 * 2
        assert UNARY[f](np.array([0.0]))[0] == 0.0
    # erf form is x * Phi(x) (standard normal CDF from scipy.stats, a different routine)
    np.testing.assert_allclose(UNARY["GELU_ERF"](x), x * scipy.stats.norm.cdf(x), rtol=1e-13, atol=1e-15)
    # tanh form approximates the erf form to < 5e-4 (Hendrycks & Gimpel)
    assert np.max(np.abs(UNARY["GELU_TANH"](x) - UNARY["GELU_ERF"](x))) < 5e-4


def test_gelu_tanh_grad_matches_finite_difference():
    g = golden("gelu_values.txt")
    assert UNARY["GELU_TANH_GRAD"](np.array([0.0]))[0] == g["gelu_grad_0"][0]
    x = np.linspace(-8, 8, 4001)
    h = 1e-5
    fd = (UNARY["GELU_TANH"](x + h) - UNARY["GELU_TANH"](x - h)) / (2 * h)
    np.testing.assert_allclose(UNARY["GELU_TANH_GRAD"](x), fd, atol=2e-9)
    # limits: gelu' -> 1 for large x, -> 0 for very negative x
    assert UNARY["GELU_TANH_GRAD"](np.array([30.0]))[0] == pytest.approx(1.0, abs=1e-12)
    assert UNARY["GELU_TANH_GRAD"](np.array([-30.0]))[0] == pytest.approx(0.0, abs=1e-12)


def test_c5_dz_is_dy_times_gelu_grad():
    spec = specs.get("C5", rows=300, cols=48)
    x = gen.generate("C5", spec)
    out = evaluate(spec, x)
    dy, z = widen(x["dy"], "BF16"), widen(x["z"], "BF16")
    # finite-difference derivative (independent of the closed-form gradient)
    h = 1e-5
    fd = (UNARY["GELU_TANH"](z + h) - UNARY["GELU_TANH"](z - h)) / (2 * h)
    np.testing.assert_allclose(out["dz"], dy * fd, atol=2e-8)
    np.testing.assert_allclose(out["db"], (dy * fd).sum(axis=0), atol=2e-6)
    np.testing.assert_allclose(out["b_new"], x["b"].astype(np.float64) - out["db"] / 128.0, rtol=1e-15)


# ---------------------------------------------------------------- figures

def test_fig5_golden():
    g = golden("fig5_power_broadcast_add.txt")
    spec = specs.get("fig5", cols=4)
    out = evaluate(spec, {"p": np.array(g["p"], np.float32),
                          "y": np.array([g["y0"], g["y1"]], np.float32)})["o"]
    np.testing.assert_array_equal(out, np.array([g["o0"], g["o1"]]))


def test_fig7a_bruteforce():
    spec = specs.get("fig7a", rows=5, cols=3)
    x = gen.generate("fig7a", spec)
    out = evaluate(spec, x, row_chunk=2)["multiply1"]
    X = x["x"].astype(np.float64)
    p2 = x["p2"].astype(np.float64)
    R, C = X.shape
    A = [[0.0] * C for _ in range(R)]
    for r in range(R):
        s = 0.0
        for c in range(C):
            s += X[r, c]
        d = s / p2[r]
        for c in range(C):
            A[r][c] = X[r, c] - d
    R2 = [sum(A[r][c] * A[r][c] for r in range(R)) for c in range(C)]
    for r in range(R):
        for c in range(C):
            assert out[r, c] == pytest.approx(A[r][c] * A[r][c] * R2[c], rel=1e-13, abs=1e-13)


# ---------------------------------------------------------------- dependent column reductions

def test_batchnorm_two_levels_invariants():
    """Training BatchNorm: mean, then variance of the centred values (two
    dependent column reductions).  Per channel the normalised output has mean 0
    and variance v/(v+eps) (closed form); mean/var match numpy's routines."""
    spec = specs.get("bn", rows=3000, cols=24)
    x = gen.generate("bn", spec)
    x["gamma"] = np.ones(24, np.float32)
    x["beta"] = np.zeros(24, np.float32)
    for chunk in (7, 512, 100000):
        out = evaluate(spec, x, row_chunk=chunk)
        X = x["x"].astype(np.float64)
        np.testing.assert_allclose(out["mean"], X.mean(axis=0), rtol=1e-13, atol=1e-15)
        v = X.var(axis=0)
        np.testing.assert_allclose(out["var"], v, rtol=1e-12)
        np.testing.assert_allclose(out["y"].mean(axis=0), 0.0, atol=1e-13)
        np.testing.assert_allclose(out["y"].var(axis=0), v / (v + 1e-5), rtol=1e-11)


def test_batchnorm_bruteforce_tiny():
    spec = specs.get("bn", rows=5, cols=2)
    x = gen.generate("bn", spec)
    out = evaluate(spec, x, row_chunk=2)
    X = x["x"].astype(np.float64)
    g, b = x["gamma"].astype(np.float64), x["beta"].astype(np.float64)
    for c in range(2):
        m = sum(X[r, c] for r in range(5)) / 5
        var = sum((X[r, c] - m) ** 2 for r in range(5)) / 5
        assert out["mean"][c] == pytest.approx(m, rel=1e-14)
        assert out["var"][c] == pytest.approx(var, rel=1e-13)
        for r in range(5):
            assert out["y"][r, c] == pytest.approx((X[r, c] - m) / math.sqrt(var + 1e-5) * g[c] + b[c],
                                                   rel=1e-12, abs=1e-13)


# ---------------------------------------------------------------- plumbing

def test_bf16_widening_golden():
    with open(os.path.join(GOLD, "bf16_bits.txt")) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            k, v = line.split(":")
            assert widen(np.array([int(k, 16)], np.uint16), "BF16")[0] == float(v)


def test_chunking_invariance():
    for name, rows, cols in (("C5", 777, 40), ("fig7a", 301, 17), ("C2", 100, 64)):
        spec = specs.get(name, rows=rows, cols=cols)
        x = gen.generate(name, spec)
        a = evaluate(spec, x, row_chunk=7)
        b = evaluate(spec, x, row_chunk=100000)
        for k in a:
            np.testing.assert_allclose(a[k], b[k], rtol=1e-13, atol=1e-13)


def test_row_and_column_subsets():
    spec = specs.get("C5", rows=600, cols=40)
    x = gen.generate("C5", spec)
    full = evaluate(spec, x)
    cols = np.array([0, 7, 39])
    sub = evaluate_columns(spec, x, cols)
    np.testing.assert_array_equal(sub["db"], full["db"][cols])
    np.testing.assert_array_equal(sub["dz"], full["dz"][:, cols])
    s3 = specs.get("C3", rows=4 * 32, cols=64)
    s3["mask"]["rows_per_segment"] = 32
    x3 = gen.generate("C3", s3)
    f3 = evaluate(s3, x3)
    rows = np.array([0, 31, 32, 77, 127])
    np.testing.assert_array_equal(evaluate_rows(s3, x3, rows)["p"], f3["p"][rows])


def test_generator_prefix_and_determinism():
    spec = specs.get("C5", rows=2 * gen.CHUNK_ROWS + 5, cols=16)
    a = gen.generate("C5", spec)
    b = gen.generate("C5", specs.get("C5", rows=100, cols=16))
    np.testing.assert_array_equal(a["dy"][:100], b["dy"])
    c = gen.generate("C5", spec, threads=1)
    np.testing.assert_array_equal(a["z"], c["z"])
    L = gen.generate("C3", specs.get("C3"))["L"]
    assert L.shape == (64,) and L[0] == 37 and L[-1] == 512 and L.min() >= 37 and L.max() <= 512
