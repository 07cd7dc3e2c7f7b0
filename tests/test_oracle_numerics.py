"""Pins for oracle/numerics.py against exact rational arithmetic (not against itself).

DESIGN.md reading R6: one correctly rounded binary op per reduce instruction. The oracle
computes bf16/fp16 ops as round_RNE(fp32(a) op fp32(b)); here the correctly rounded
result of the *exact* rational a op b is computed independently (Fractions and an
explicit round-half-even), so a wrong shift, a wrong tie rule or double rounding fails.
"""
import math
import struct
from fractions import Fraction

import numpy as np
import pytest

from oracle import numerics as nm

pytestmark = pytest.mark.filterwarnings("ignore::RuntimeWarning")


def _bf16_bits_to_fraction(u):
    f = struct.unpack("<f", struct.pack("<I", int(u) << 16))[0]
    return Fraction(f)


def _round_exact(fr, mant_bits, emin, emax):
    """Correctly rounded (RNE) value of rational fr in a binary format with `mant_bits`
    fraction bits, minimum normal exponent emin; returns a Fraction or +-inf."""
    if fr == 0:
        return Fraction(0)
    neg = fr < 0
    a = -fr if neg else fr
    e = a.numerator.bit_length() - a.denominator.bit_length()
    if Fraction(2) ** e > a:
        e -= 1
    if Fraction(2) ** (e + 1) <= a:
        e += 1
    e = max(e, emin)
    ulp = Fraction(2) ** (e - mant_bits)
    q = a / ulp
    n = q.numerator // q.denominator
    rem = q - n
    if rem > Fraction(1, 2) or (rem == Fraction(1, 2) and n % 2 == 1):
        n += 1
    v = n * ulp
    if v >= Fraction(2) ** (emax + 1):
        return -math.inf if neg else math.inf
    return -v if neg else v


def _bf16_from_value(v):
    if v in (math.inf, -math.inf):
        return 0xFF80 if v < 0 else 0x7F80
    bits = struct.unpack("<I", struct.pack("<f", float(v)))[0]
    assert bits & 0xFFFF == 0
    return bits >> 16


def _random_bf16(rng, n):
    # sign, exponent spread over most of the range, random mantissa, plus subnormals
    exp = rng.integers(1, 254, n)
    exp[: n // 10] = 0
    man = rng.integers(0, 128, n)
    sign = rng.integers(0, 2, n)
    return ((sign << 15) | (exp << 7) | man).astype(np.uint16)


@pytest.mark.parametrize("op", ["sum", "prod"])
def test_bf16_single_rounding_matches_exact_rational(op):
    rng = np.random.default_rng(1)
    a = _random_bf16(rng, 3000)
    # bias b's exponent near a's so that sums actually round (both far and near cases)
    b = _random_bf16(rng, 3000)
    b[:1500] = (a[:1500] & 0xFF80) ^ (rng.integers(0, 128, 1500).astype(np.uint16))
    got = nm.reduce(a, b, op, "bfloat16")
    for x, y, g in zip(a, b, got):
        fx, fy = _bf16_bits_to_fraction(x), _bf16_bits_to_fraction(y)
        exact = fx + fy if op == "sum" else fx * fy
        want = _round_exact(exact, 7, -126, 127)
        if want == 0:
            assert (int(g) & 0x7FFF) == 0
            continue
        assert int(g) == _bf16_from_value(want), (hex(x), hex(y), hex(int(g)))


@pytest.mark.parametrize("op", ["sum", "prod"])
def test_fp16_single_rounding_matches_exact_rational(op):
    rng = np.random.default_rng(2)
    bits = rng.integers(0, 0x7C00, 6000).astype(np.uint16)       # finite, incl. subnormals
    bits |= (rng.integers(0, 2, 6000).astype(np.uint16) << 15)
    v = bits.view(np.float16)
    a, b = v[:3000], v[3000:]
    got = nm.reduce(a, b, op, "float16")
    for x, y, g in zip(a, b, got):
        exact = Fraction(float(x)) + Fraction(float(y)) if op == "sum" else Fraction(float(x)) * Fraction(float(y))
        want = _round_exact(exact, 10, -14, 15)
        if want == 0:
            assert float(g) == 0.0
        else:
            assert float(g) == float(want), (x, y, g, want)


def test_bf16_narrowing_special_values():
    f = np.array([1.0, -2.5, np.inf, -np.inf, 3.4028234663852886e38, 1.00390625, 1.01171875, 0.0],
                 dtype=np.float32)
    got = nm.f32_to_bf16(f)
    # 1.00390625 = 1 + 2^-8 is a tie -> even (1.0); 1.01171875 = 1 + 3*2^-8 tie -> 1 + 2^-6
    assert list(got) == [0x3F80, 0xC020, 0x7F80, 0xFF80, 0x7F80, 0x3F80, 0x3F82, 0x0000]
    assert nm.f32_to_bf16(np.array([np.nan], dtype=np.float32))[0] == 0x7FC0
    assert nm.bf16_to_f32(np.array([0x3F80, 0xC020], dtype=np.uint16)).tolist() == [1.0, -2.5]


def test_integer_wraparound_and_minmax():
    a = np.array([2**31 - 1, -5, 7], dtype=np.int32)
    b = np.array([1, 3, -9], dtype=np.int32)
    assert nm.reduce(a, b, "sum", "int32").tolist() == [-2**31, -2, -2]
    assert nm.reduce(a, b, "max", "int32").tolist() == [2**31 - 1, 3, 7]
    assert nm.reduce(a, b, "min", "int32").tolist() == [1, -5, -9]
    assert nm.reduce(np.array([2**16], np.int32), np.array([2**16], np.int32), "prod", "int32").tolist() == [0]
    u = np.array([0xFFFFFFFF], dtype=np.uint32)
    assert nm.reduce(u, np.array([2], np.uint32), "sum", "uint32").tolist() == [1]
