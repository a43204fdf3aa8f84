"""Host check of the seismic kernel's division scheme (csrc/seismic.cu
dz_point / div_fast / div_range), in exact arithmetic: for every difference d
whose exponent lies in the per-launch range the kernel takes the fast path
for, q = d*y, then two corrections q += fma(-q, h, d)*y with y = RN(1/h),
equals the IEEE quotient d/h bit for bit; everything outside the range (zeros,
subnormals, non-finite values, extreme quotients) takes the IEEE division in
the kernel.  fma is evaluated exactly with fractions (one rounding), so this
pins the arithmetic the GPU path relies on, independently of the GPU."""
import math
import random
import struct
from fractions import Fraction

import pytest


def fma(a, b, c):
    return float(Fraction(a) * Fraction(b) + Fraction(c))  # correctly rounded


def div_fast(d, h, y):
    q0 = d * y
    q = fma(fma(-q0, h, d), y, q0)
    return fma(fma(-q, h, d), y, q)


def ebits(x):
    return (struct.unpack("<Q", struct.pack("<d", x))[0] >> 32) & 0x7FF00000


def div_range(h):  # the host side (seismic.cu div_range)
    _, eh = math.frexp(h)
    e = eh + 1022
    lo, hi = max(64, e - 958), min(1983, e + 959)
    if lo > hi or not (2.0 ** -900 <= abs(h) <= 2.0 ** 900):
        return 0xFFFFFFFF, 0
    return lo << 20, (hi - lo) << 20


def fast_ok(d, rng):
    lo, span = rng
    return ((ebits(d) - lo) & 0xFFFFFFFF) <= span


@pytest.mark.parametrize("seed", [1, 2])
def test_fast_division_bit_identical_in_range(seed):
    r = random.Random(seed)
    hs = [0.37, 0.01, 1.0 / 3.0, 3.0, 1e-7, 12345.678, 2.0 ** -20, -2.5,
          2.0 - 2.0 ** -52, 1.0 + 2.0 ** -52]
    fast = 0
    for t in range(6000):
        h = r.choice(hs + [r.uniform(0.01, 100.0), r.uniform(1, 2) * 2.0 ** r.randint(-890, 890)])
        y = 1.0 / h
        rng = div_range(h)
        d = r.gauss(0, 1) * 2.0 ** r.randint(-1074, 1023)
        if r.random() < 0.4:
            d = r.gauss(0, 1) * 2.0 ** r.randint(-40, 40)
        if not math.isfinite(d) or not fast_ok(d, rng):
            continue
        fast += 1
        q = div_fast(d, h, y)
        assert struct.pack("<d", q) == struct.pack("<d", d / h), (d, h, q, d / h)
    assert fast > 3000


def test_range_excludes_the_unsafe_values():
    rng = div_range(0.37)
    for d in (0.0, -0.0, 5e-324, 2.0 ** -1030, math.inf, -math.inf, math.nan, 1.7e308):
        assert not fast_ok(d, rng)
    for d in (1.0, -3.5, 1e-250, 1e250):
        assert fast_ok(d, rng)
    assert not fast_ok(1.0, div_range(1e-300))  # h outside [2^-900, 2^900]: never fast


def test_subnormal_difference_is_why_the_range_exists():
    # the bare correction form is NOT exact for every subnormal difference
    # (found by the same emulation); the range test routes them to IEEE
    bad = 0
    r = random.Random(5)
    for _ in range(4000):
        h = r.uniform(1, 2) * 2.0 ** r.randint(-300, -30)
        d = r.gauss(0, 1) * 2.0 ** r.randint(-1074, -1023)
        if d == 0.0:
            continue
        if div_fast(d, h, 1.0 / h) != d / h:
            bad += 1
        assert not fast_ok(d, div_range(h))
    assert bad > 0
