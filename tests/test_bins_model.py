"""Host model of the exact binned column sums (reading R23,
kernels/astitch_device.cuh: bins_add / bins_merge / bins_value_d and the
precise variant bins_add_p / bins_merge_p / bins_value_p), checked against
exact rational arithmetic:

* the total does not depend on the order of the deposits nor on how they
  are split across accumulators that are merged later (the property the
  tma_sweep relies on: any CTA may take any tile);
* it equals the sum of every deposit truncated (toward zero) at the bottom of
  the column's final window, so the error is below n * 2^-32 (fp32 bins) /
  n * 2^-48 (precise bins) of the largest deposit;
* +-inf / NaN deposits give the IEEE sum of the non-finite ones.

The model mirrors the device code operation by operation (integers are
Python ints: the device's int64 bins cannot overflow at these counts).
"""

from fractions import Fraction
import math
import struct

import numpy as np
import pytest

EMPTY = -1000


def fsum32(a, b):
    """fp32 a + b (inf - inf = NaN, no warning): the device's side sum."""
    with np.errstate(invalid="ignore"):
        return float(np.float32(a) + np.float32(b))


# ---------------------------------------------------------------- fp32 bins
def f32_bits(x):
    return struct.unpack("<I", struct.pack("<f", x))[0]


class Bins:
    """Two 32-bit-aligned bins of a 64-bit window on the scale 2^-160."""

    def __init__(self):
        self.J, self.hi, self.lo, self.sp = EMPTY, 0, 0, 0.0

    def add(self, x):
        u = f32_bits(x)
        a = u & 0x7FFFFFFF
        if a >= 0x7F800000:
            self.sp = fsum32(self.sp, x)
            return
        e = a >> 23
        need = (max(e, 1) + 1) >> 5 if a else EMPTY
        if need > self.J:
            self.lo = self.hi if need == self.J + 1 else 0
            self.hi = 0
            self.J = need
        m = (u & 0x7FFFFF) | (0x800000 if e else 0)
        d = min(max(e, 1) + 10 - 32 * self.J, 40)
        v = (m << d) if d >= 0 else ((m >> -d) if d > -24 else 0)
        vl, vh = v & 0xFFFFFFFF, v >> 32
        if u >> 31:
            self.lo -= vl
            self.hi -= vh
        else:
            self.lo += vl
            self.hi += vh

    def merge(self, o):
        self.sp = fsum32(self.sp, o.sp)
        if o.J > self.J:
            self.lo = self.hi if o.J == self.J + 1 else 0
            self.hi = 0
            self.J = o.J
        if o.J == self.J:
            self.hi += o.hi
            self.lo += o.lo
        elif o.J == self.J - 1:
            self.lo += o.hi

    def exact(self):
        if self.J == EMPTY:
            return Fraction(0)
        return Fraction(self.hi) * Fraction(2) ** (32 * (self.J + 1) - 160) + Fraction(self.lo) * Fraction(2) ** (32 * self.J - 160)

    def value(self):
        if self.sp != 0.0 or math.isnan(self.sp):
            return self.sp
        if self.J == EMPTY:
            return 0.0
        return math.ldexp(float(self.hi), 32 * (self.J + 1) - 160) + math.ldexp(float(self.lo), 32 * self.J - 160)


# ---------------------------------------------------------------- fp64 (precise) bins
def f64_bits(x):
    return struct.unpack("<Q", struct.pack("<d", x))[0]


class BinsP:
    """Four 16-bit-aligned bins of a 64-bit window on the scale 2^-1100."""

    def __init__(self):
        self.J, self.b, self.sp = EMPTY, [0, 0, 0, 0], 0.0

    def _shift(self, need):
        t = need - self.J
        self.b = [self.b[k + t] if k + t < 4 else 0 for k in range(4)]
        self.J = need

    def add(self, x):
        u = f64_bits(x)
        e = (u >> 52) & 0x7FF
        if e == 0x7FF:
            self.sp = fsum32(self.sp, x)
            return
        mn = u & 0xFFFFFFFFFFFFF
        if not (mn | e):
            return
        bi = max(e, 1) + 25
        need = (bi + 4) >> 4
        if need > self.J:
            if self.J == EMPTY or need - self.J >= 4:
                self.b, self.J = [0, 0, 0, 0], need
            else:
                self._shift(need)
        m = mn | ((1 << 52) if e else 0)
        d = min(bi - 16 * self.J, 11)
        v = (m << d) if d >= 0 else ((m >> -d) if d > -53 else 0)
        for q in range(4):
            sl = (v >> (16 * q)) & 0xFFFF
            self.b[q] += -sl if u >> 63 else sl

    def merge(self, o):
        self.sp = fsum32(self.sp, o.sp)
        if o.J == EMPTY:
            return
        if self.J == EMPTY or o.J - self.J >= 4:
            if o.J > self.J:
                self.b, self.J = [0, 0, 0, 0], o.J
        elif o.J > self.J:
            self._shift(o.J)
        t = self.J - o.J
        for k in range(4):
            if k + t < 4:
                self.b[k] += o.b[k + t]

    def exact(self):
        if self.J == EMPTY:
            return Fraction(0)
        return sum(Fraction(self.b[k]) * Fraction(2) ** (16 * (self.J + k) - 1100) for k in range(4))


def trunc_at(x, unit):
    """x truncated toward zero to a multiple of `unit` (exact)."""
    q = Fraction(x) / unit
    return (math.floor(q) if q >= 0 else math.ceil(q)) * unit


def deposits(rng, n, kind):
    if kind == "normal":
        return [float(np.float32(v)) for v in rng.standard_normal(n) * 10.0 ** rng.integers(-3, 4, n)]
    if kind == "wide":      # exponents across most of the fp32 range, both signs
        return [float(np.float32(np.ldexp(rng.uniform(0.5, 1.0) * rng.choice([-1, 1]), int(rng.integers(-140, 120)))))
                for _ in range(n)]
    if kind == "cancel":    # large values that cancel, small values underneath
        big = [float(np.float32(3e37)), float(np.float32(-3e37))] * (n // 8)
        return big + [float(np.float32(v)) for v in rng.standard_normal(n - len(big))]
    if kind == "subnormal":
        return [float(np.float32(v)) for v in rng.standard_normal(n) * 1e-40] + [0.0, -0.0]
    raise ValueError(kind)


@pytest.mark.parametrize("kind", ["normal", "wide", "cancel", "subnormal"])
@pytest.mark.parametrize("seed", range(4))
def test_fp32_bins_order_and_partition_independent(kind, seed):
    rng = np.random.default_rng(seed)
    xs = deposits(rng, 300, kind)
    ref = Bins()
    for x in xs:
        ref.add(x)
    for trial in range(4):
        perm = rng.permutation(len(xs))
        parts = [Bins() for _ in range(int(rng.integers(1, 9)))]
        for i in perm:
            parts[int(rng.integers(0, len(parts)))].add(xs[i])
        # merge in a random order and a random tree shape
        while len(parts) > 1:
            i, j = sorted(rng.choice(len(parts), 2, replace=False))
            parts[i].merge(parts[j])
            parts.pop(j)
        got = parts[0]
        assert (got.J, got.hi, got.lo) == (ref.J, ref.hi, ref.lo), (kind, seed, trial)
        assert got.value() == ref.value() or (math.isnan(got.value()) and math.isnan(ref.value()))


@pytest.mark.parametrize("kind", ["normal", "wide", "cancel", "subnormal"])
def test_fp32_bins_equal_truncated_sum(kind):
    """Total = sum of each deposit truncated at the final window's bottom;
    error <= n * 2^-32 * max|x| (>= 32 bits kept below the largest deposit)."""
    rng = np.random.default_rng(7)
    xs = deposits(rng, 400, kind)
    b = Bins()
    for x in xs:
        b.add(x)
    unit = Fraction(2) ** (32 * b.J - 160)
    assert b.exact() == sum(trunc_at(x, unit) for x in xs)
    exact = sum(Fraction(x) for x in xs)
    mx = max(abs(Fraction(x)) for x in xs)
    assert abs(b.exact() - exact) <= len(xs) * mx * Fraction(2) ** -32
    # the device value is one fp64 rounding of the exact total (then fp32)
    assert abs(Fraction(b.value()) - b.exact()) <= abs(b.exact()) * Fraction(2) ** -52 + Fraction(2) ** -1074


def test_fp32_bins_nonfinite():
    b = Bins()
    for x in [1.0, float("inf"), 2.0]:
        b.add(x)
    assert b.value() == float("inf")
    b.add(float("-inf"))
    assert math.isnan(b.value())
    c = Bins()
    c.add(float("nan"))
    c.add(5.0)
    assert math.isnan(c.value())


@pytest.mark.parametrize("seed", range(4))
def test_precise_bins_order_independent_and_48_bits(seed):
    """fp64 tile partials of a column whose mean is 3e6 x its spread (the R7c
    case): 4 x 16-bit bins keep >= 48 bits below the largest deposit, so the
    mean survives, and any order / partition gives the same bins."""
    rng = np.random.default_rng(100 + seed)
    xs = [float(16 * 3.0e4 + v) for v in rng.standard_normal(500) * 0.01]   # 16-row partials
    xs += [float(np.ldexp(rng.uniform(0.5, 1), int(rng.integers(-60, 60)))) * rng.choice([-1, 1]) for _ in range(50)]
    ref = BinsP()
    for x in xs:
        ref.add(x)
    for trial in range(3):
        parts = [BinsP() for _ in range(int(rng.integers(1, 7)))]
        for i in rng.permutation(len(xs)):
            parts[int(rng.integers(0, len(parts)))].add(xs[i])
        while len(parts) > 1:
            i, j = sorted(rng.choice(len(parts), 2, replace=False))
            parts[i].merge(parts[j])
            parts.pop(j)
        assert (parts[0].J, parts[0].b) == (ref.J, ref.b)
    exact = sum(Fraction(x) for x in xs)
    mx = max(abs(Fraction(x)) for x in xs)
    assert abs(ref.exact() - exact) <= len(xs) * mx * Fraction(2) ** -48
    unit = Fraction(2) ** (16 * ref.J - 1100)
    assert ref.exact() == sum(trunc_at(x, unit) for x in xs)
