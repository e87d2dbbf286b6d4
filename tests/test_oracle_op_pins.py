"""Pins for every element-wise op and input widening of the fp64 oracle.

Each op is evaluated THROUGH ``oracle.evaluate`` on a tiny spec (so the
dispatch table entry the parity tests use is the one pinned) and checked
against closed forms, textbook constants (tests/golden/unary_values.txt,
Abramowitz & Stegun), exact special cases, identities that a plausible slip
breaks (a dropped minus sign in SIGMOID gives sigmoid(ln 3) = 1/4, a swapped
SUB/DIV operand gives -2 / 1.5, MAX <-> MIN fails the brute force), and
derivative relations checked by finite differences.
"What pins each part".  Also: RMAX propagates NaN (reading R12), and F16
widening against IEEE binary16 bit patterns.
"""

import math
import os

import numpy as np
import pytest

from oracle import evaluate, widen

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def golden(name):
    d = {}
    with open(os.path.join(GOLD, name)) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            k, v = line.split(":", 1)
            d[k.strip()] = float(v)
    return d


G = golden("unary_values.txt")


def un(op, x):
    """Evaluate one unary op through the oracle on a [1, n] F32 input (every
    test value is exactly representable in fp32)."""
    x = np.atleast_1d(np.asarray(x, dtype=np.float32))
    spec = {"name": "pin", "rows": 1, "cols": x.size, "inputs": [("a", "FULL", "F32")], "mask": None,
            "ops": [("y", "unary", op, "a")], "outputs": [("y", "F32")]}
    return evaluate(spec, {"a": x[None, :]})["y"][0]


def bi(op, a, b):
    a = np.atleast_1d(np.asarray(a, dtype=np.float32))
    b = np.atleast_1d(np.asarray(b, dtype=np.float32))
    spec = {"name": "pin", "rows": 1, "cols": a.size,
            "inputs": [("a", "FULL", "F32"), ("b", "FULL", "F32")], "mask": None,
            "ops": [("y", "binary", op, "a", "b")], "outputs": [("y", "F32")]}
    return evaluate(spec, {"a": a[None, :], "b": b[None, :]})["y"][0]


X = np.linspace(-5.0, 5.0, 401).astype(np.float32)      # exact fp32 grid points
XP = np.linspace(0.05, 20.0, 400).astype(np.float32)    # positive grid


# ------------------------------------------------------------------ unary

def test_neg_abs():
    assert un("NEG", 3.0)[0] == -3.0 and un("NEG", -0.5)[0] == 0.5
    np.testing.assert_array_equal(un("NEG", X) + X.astype(np.float64), 0.0)
    a = un("ABS", X)
    assert (a >= 0).all() and un("ABS", -2.5)[0] == 2.5
    for xi, ai in zip(X, a):                            # brute force: |x| = x if x >= 0 else -x
        assert ai == (float(xi) if xi >= 0 else -float(xi))


def test_exp():
    assert un("EXP", 0.0)[0] == 1.0
    assert un("EXP", 1.0)[0] == pytest.approx(G["e"], rel=1e-15)
    assert un("EXP", -1.0)[0] == pytest.approx(1.0 / G["e"], rel=1e-15)
    # exp(a) * exp(b) = exp(a + b) on exactly representable a, b, a + b
    a = np.array([0.5, 1.25, -3.0, 2.0], np.float32)
    b = np.array([0.25, -0.75, 1.5, 2.0], np.float32)
    np.testing.assert_allclose(un("EXP", a) * un("EXP", b), un("EXP", a + b), rtol=1e-14)
    assert un("EXP", 2.0)[0] == pytest.approx(G["e"] ** 2, rel=1e-15)


def test_log():
    assert un("LOG", 1.0)[0] == 0.0
    assert un("LOG", 2.0)[0] == pytest.approx(G["ln2"], rel=1e-15)
    assert un("LOG", 8.0)[0] == pytest.approx(3 * G["ln2"], rel=1e-15)
    assert un("LOG", 0.25)[0] == pytest.approx(-2 * G["ln2"], rel=1e-15)
    # log(e) = 1 on the exact product: log(x * y) = log x + log y for powers of two
    np.testing.assert_allclose(un("LOG", XP * 4.0), un("LOG", XP) + 2 * G["ln2"], rtol=1e-13, atol=1e-15)
    # derivative: d/dx log x = 1/x (central difference on the exact grid)
    h = np.float32(2.0 ** -10)
    fd = (un("LOG", XP + h) - un("LOG", XP - h)) / (2 * float(h))
    np.testing.assert_allclose(fd, 1.0 / XP.astype(np.float64), rtol=5e-4)  # O(h^2/x^2) FD error
    assert math.isnan(un("LOG", -1.0)[0]) and un("LOG", 0.0)[0] == -math.inf


def test_sqrt_rsqrt_rcp():
    assert un("SQRT", 4.0)[0] == 2.0 and un("SQRT", 0.0)[0] == 0.0
    assert un("SQRT", 2.0)[0] == pytest.approx(G["sqrt2"], rel=1e-16)
    s = un("SQRT", XP)
    assert (s > 0).all()
    np.testing.assert_allclose(s * s, XP.astype(np.float64), rtol=1e-15)
    assert un("RSQRT", 4.0)[0] == 0.5 and un("RSQRT", 0.25)[0] == 2.0
    r = un("RSQRT", XP)
    np.testing.assert_allclose(r * r * XP.astype(np.float64), 1.0, rtol=1e-15)
    assert un("RCP", 4.0)[0] == 0.25 and un("RCP", -2.0)[0] == -0.5
    np.testing.assert_allclose(un("RCP", X[X != 0]) * X[X != 0].astype(np.float64), 1.0, rtol=1e-15)


def test_tanh():
    assert un("TANH", 0.0)[0] == 0.0
    assert un("TANH", 1.0)[0] == pytest.approx(G["tanh_1"], rel=1e-15)
    # tanh(ln(3)/2) = 1/2: the input ln(3)/2 is not an fp32 value, so go via x = fp32(ln 3 / 2)
    x = np.float32(math.log(3.0) / 2)
    e2 = math.exp(2 * float(x))
    assert un("TANH", x)[0] == pytest.approx((e2 - 1) / (e2 + 1), rel=1e-14)
    assert un("TANH", x)[0] == pytest.approx(G["tanh_half_ln3"], rel=1e-7)
    t = un("TANH", X)
    np.testing.assert_array_equal(t, -un("TANH", -X))    # odd
    assert (np.abs(t) < 1).all() or (np.abs(t) <= 1).all()
    # tanh' = 1 - tanh^2
    h = np.float32(2.0 ** -10)
    fd = (un("TANH", X + h) - un("TANH", X - h)) / (2 * float(h))
    np.testing.assert_allclose(fd, 1 - t * t, atol=2e-6)


def test_erf():
    assert un("ERF", 0.0)[0] == 0.0
    assert un("ERF", 1.0)[0] == pytest.approx(G["erf_1"], rel=1e-15)
    assert un("ERF", 0.5)[0] == pytest.approx(G["erf_half"], rel=1e-15)
    np.testing.assert_array_equal(un("ERF", X), -un("ERF", -X))
    assert un("ERF", 30.0)[0] == 1.0
    # erf' = 2/sqrt(pi) exp(-x^2)
    h = np.float32(2.0 ** -10)
    fd = (un("ERF", X + h) - un("ERF", X - h)) / (2 * float(h))
    Xd = X.astype(np.float64)
    np.testing.assert_allclose(fd, 2 / math.sqrt(math.pi) * np.exp(-Xd * Xd), atol=2e-6)


def test_sigmoid():
    assert un("SIGMOID", 0.0)[0] == 0.5
    s = un("SIGMOID", X)
    np.testing.assert_allclose(s + un("SIGMOID", -X), 1.0, rtol=0, atol=1e-15)   # symmetry
    assert (np.diff(s) > 0).all()                                                 # increasing
    x = np.float32(math.log(3.0))
    assert un("SIGMOID", x)[0] == pytest.approx(G["sigmoid_ln3"], rel=1e-7)       # 3/4, not 1/4
    # sigma' = sigma (1 - sigma)
    h = np.float32(2.0 ** -10)
    fd = (un("SIGMOID", X + h) - un("SIGMOID", X - h)) / (2 * float(h))
    np.testing.assert_allclose(fd, s * (1 - s), atol=1e-7)
    # relation to tanh: sigma(2x) = (1 + tanh x) / 2
    np.testing.assert_allclose(un("SIGMOID", 2 * X), 0.5 * (1 + un("TANH", X)), atol=1e-15)


# ------------------------------------------------------------------ binary

def test_binary_operand_order_and_values():
    a = np.array([5.0, -3.0, 6.0, 0.5], np.float32)
    b = np.array([3.0, 2.0, -1.5, 0.25], np.float32)
    np.testing.assert_array_equal(bi("ADD", a, b), [8.0, -1.0, 4.5, 0.75])
    np.testing.assert_array_equal(bi("SUB", a, b), [2.0, -5.0, 7.5, 0.25])     # a - b, not b - a
    np.testing.assert_array_equal(bi("MUL", a, b), [15.0, -6.0, -9.0, 0.125])
    np.testing.assert_array_equal(bi("DIV", a, b), [5 / 3, -1.5, -4.0, 2.0])   # a / b, not b / a
    np.testing.assert_array_equal(bi("POW", np.array([2.0, -2.0, 4.0, 9.0], np.float32),
                                     np.array([3.0, 3.0, 0.5, 0.5], np.float32)), [8.0, -8.0, 2.0, 3.0])


def test_max_min_bruteforce():
    rng = np.random.default_rng(3)
    a = rng.integers(-4, 5, 200).astype(np.float32)
    b = rng.integers(-4, 5, 200).astype(np.float32)
    mx, mn = bi("MAX", a, b), bi("MIN", a, b)
    for ai, bi_, x, n in zip(a, b, mx, mn):
        assert x == (ai if ai >= bi_ else bi_)
        assert n == (ai if ai <= bi_ else bi_)
    np.testing.assert_array_equal(mx + mn, a.astype(np.float64) + b)          # {max, min} = {a, b}


def test_pow_integer_exponent_negative_base():
    # R11: x^3 with a negative base is a product, not exp(3 log x) (= NaN)
    x = np.array([-2.0, -0.5, 3.0], np.float32)
    three = np.full(3, 3.0, np.float32)
    np.testing.assert_array_equal(bi("POW", x, three), x.astype(np.float64) ** 3)
    spec = {"name": "pin", "rows": 1, "cols": 3, "inputs": [("a", "FULL", "F32")], "mask": None,
            "ops": [("k", "const", 3.0), ("y", "binary", "POW", "a", "k")], "outputs": [("y", "F32")]}
    np.testing.assert_array_equal(evaluate(spec, {"a": x[None, :]})["y"][0], [-8.0, -0.125, 27.0])


# ------------------------------------------------------------------ R12, widening

@pytest.mark.parametrize("axis", ["ROW", "COL"])
def test_rmax_propagates_nan(axis):
    """Reading R12: RMAX propagates NaN (a NaN anywhere in the reduced set
    makes the result NaN); other rows/columns are unaffected."""
    x = np.arange(12, dtype=np.float32).reshape(3, 4)
    x[1, 2] = np.nan
    spec = {"name": "pin", "rows": 3, "cols": 4, "inputs": [("x", "FULL", "F32")], "mask": None,
            "ops": [("m", "reduce", "RMAX", axis, "x")], "outputs": [("m", "F32")]}
    m = evaluate(spec, {"x": x})["m"]
    if axis == "ROW":
        assert m[0] == 3.0 and math.isnan(m[1]) and m[2] == 11.0
    else:
        assert m[0] == 8.0 and m[1] == 9.0 and math.isnan(m[2]) and m[3] == 11.0


def test_f16_widening_golden():
    with open(os.path.join(GOLD, "f16_bits.txt")) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            k, v = line.split(":")
            bits = np.array([int(k, 16)], np.uint16).view(np.float16)
            w = widen(bits, "F16")[0]
            assert w == float(v) and math.copysign(1.0, w) == math.copysign(1.0, float(v))
