"""Independent helpers for pinning the oracle (pure Python, exact arithmetic where it matters).

Nothing here imports oracle/ or the CUDA path. mix64 is pinned to the published splitmix64
vectors in tests/golden/splitmix64_seed0.json before anything relies on it.
"""
from __future__ import annotations

import json
import os
import struct
from fractions import Fraction

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")
M64 = (1 << 64) - 1
DELIMS = b" \t\n\x0b\x0c\r"


def golden(name: str):
    with open(os.path.join(GOLDEN, name)) as f:
        return json.load(f)


def mix64(x: int) -> int:
    x ^= x >> 30
    x = (x * 0xBF58476D1CE4E5B9) & M64
    x ^= x >> 27
    x = (x * 0x94D049BB133111EB) & M64
    x ^= x >> 31
    return x


def f32(v: float) -> float:
    return struct.unpack("<f", struct.pack("<f", v))[0]


def round_f32(q: Fraction) -> Fraction:
    """Round an exact rational to the nearest fp32 (ties to even); normal range only."""
    if q == 0:
        return Fraction(0)
    sign = -1 if q < 0 else 1
    a = abs(q)
    e = a.numerator.bit_length() - a.denominator.bit_length()
    # find e with 2^23 <= a / 2^e < 2^24
    while a / Fraction(2) ** e >= 2 ** 24:
        e += 1
    while a / Fraction(2) ** e < 2 ** 23:
        e -= 1
    m = a / Fraction(2) ** e
    fl = m.numerator // m.denominator
    rem = m - fl
    if rem > Fraction(1, 2) or (rem == Fraction(1, 2) and fl % 2 == 1):
        fl += 1
    return sign * Fraction(fl) * Fraction(2) ** e


def fmaf_exact(a: Fraction, b: Fraction, c: Fraction) -> Fraction:
    """fmaf: a*b + c with a single rounding to fp32."""
    return round_f32(a * b + c)


def sub_f32(a: Fraction, b: Fraction) -> Fraction:
    return round_f32(a - b)


def words_of_record(rec: bytes) -> list[bytes]:
    """Maximal runs of non-delimiter bytes (bytes.split() uses exactly the C-locale isspace set)."""
    return rec.split()
