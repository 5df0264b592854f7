"""Exact-arithmetic helpers for the tests (Fractions; no oracle code).

Correct rounding of an exact rational to binary32 / binary16 with ties to even,
written from IEEE 754 (normal and subnormal quanta).  Used to pin the oracle's
floating-point results against exact mathematics, independently of the C code.
"""
from fractions import Fraction

import numpy as np


def _round_fraction(q: Fraction, mant_bits: int, emin_normal: int, emax: int):
    if q == 0:
        return Fraction(0), False
    a = abs(q)
    e = a.numerator.bit_length() - a.denominator.bit_length()
    if Fraction(2) ** e > a:
        e -= 1
    if Fraction(2) ** (e + 1) <= a:
        e += 1
    qexp = max(e, emin_normal) - mant_bits
    scaled = a / (Fraction(2) ** qexp)
    n = scaled.numerator // scaled.denominator
    rem = scaled - n
    if rem > Fraction(1, 2) or (rem == Fraction(1, 2) and n % 2 == 1):
        n += 1
    val = Fraction(n) * Fraction(2) ** qexp
    overflow = val >= Fraction(2) ** (emax + 1)
    return (val if q > 0 else -val), overflow


def to_f32(q: Fraction) -> np.float32:
    """RNE(q) in binary32 (24-bit significand, emin -126)."""
    v, ovf = _round_fraction(Fraction(q), 23, -126, 127)
    if ovf:
        return np.float32(np.inf if q > 0 else -np.inf)
    return np.float32(float(v))


def to_f16(q: Fraction) -> np.float16:
    """RNE(q) in binary16 (11-bit significand, emin -14)."""
    v, ovf = _round_fraction(Fraction(q), 10, -14, 15)
    if ovf:
        return np.float16(np.inf if q > 0 else -np.inf)
    return np.float16(float(v))


def frac(x) -> Fraction:
    """Exact rational value of a finite float (numpy or Python)."""
    return Fraction(float(x))


def ulp32(x) -> Fraction:
    """Unit in the last place of binary32 x (exact)."""
    x = np.float32(x)
    a = abs(float(x))
    if a == 0:
        return Fraction(2) ** -149
    e = int(np.floor(np.log2(a)))
    if Fraction(2) ** e > Fraction(a):
        e -= 1
    if Fraction(2) ** (e + 1) <= Fraction(a):
        e += 1
    return Fraction(2) ** (max(e, -126) - 23)
