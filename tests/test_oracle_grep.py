"""Pins for oracle O2 (grep/filter; MCA analogue PAPER.md:965-978)."""
import struct

import numpy as np
import pytest

import gen
import oracle


def rec(key: bytes, payload: bytes = b"", i: int = 0) -> bytes:
    k = key[:32].ljust(32, b"\x00") if len(key) < 32 else key[:32]
    return struct.pack("<IIQ", 48 + len(payload), 0, i) + k + payload


def pack(recs):
    buf = b"".join(recs)
    off = np.cumsum([0] + [len(r) for r in recs[:-1]]).astype(np.uint64)
    return buf, off


def brute(buf: bytes, off, pat: bytes):
    out = []
    for i, s in enumerate(off):
        key = buf[int(s) + 16: int(s) + 48].split(b"\x00")[0]
        if key.find(pat) >= 0:
            out.append(i)
    return out


def test_adversarial_catalogue():
    recs = [
        rec(b"bigkxxxx"),                       # match at position 0
        rec(b"xxxxbigk"),                       # match at kl-4
        rec(b"a" * 28 + b"bigk"),               # 32-byte key, no NUL, match at the end
        rec(b"big\x00k"),                       # bytes after the first NUL must not complete a match
        rec(b"bi"),                             # pattern longer than the key
        rec(b"xbigkx", payload=b"bigkbigk"),    # payload matches are not key matches
        rec(b"nothing here", payload=b"zz"),
        rec(b""),                               # empty key
    ]
    buf, off = pack(recs)
    got = oracle.grep(buf, off, b"bigk")
    assert list(got) == brute(buf, off, b"bigk") == [0, 1, 2, 5]


def test_empty_pattern_and_impossible_pattern():
    buf, off = pack([rec(b"abc"), rec(b""), rec(b"q" * 32)])
    assert list(oracle.grep(buf, off, b"")) == [0, 1, 2]
    assert list(oracle.grep(buf, off, b"x" * 33)) == []


def test_first_offset_and_short_record_error():
    buf, off = pack([rec(b"bigk"), rec(b"nope"), rec(b"zbigk")])
    assert list(oracle.grep(buf, off, b"bigk", first=1000)) == [1000, 1002]
    bad = b"\x00" * 40
    with pytest.raises(ValueError):
        oracle.grep(bad, np.zeros(1, np.uint64), b"a")


def test_generated_vs_brute_force_and_planted():
    buf, off = gen.grep_records(max_bytes=1 << 20)
    b = buf.tobytes()
    got = oracle.grep(buf, off, b"bigk")
    assert list(got) == brute(b, off, b"bigk")
    # every planted record (p = 1/100, gen stream 4) must match; unplanted matches are rare
    planted = [i for i in range(len(off)) if gen.R(gen.SEED_GREP, 4, i) % 100 == 0]
    assert set(planted) <= set(int(v) for v in got)
    assert len(got) <= len(planted) + 5
    # always-true pattern (every key has >= 8 lowercase letters, so "" and single letters)
    assert len(oracle.grep(buf, off, b"")) == len(off)


def test_generator_record_format():
    buf, off = gen.grep_records(n=2000)
    b = buf.tobytes()
    ends = list(off[1:]) + [len(b)]
    for i in range(0, 2000, 97):
        s = int(off[i])
        ln, _, rid = struct.unpack_from("<IIQ", b, s)
        assert ln == int(ends[i]) - s and 48 <= ln <= 464 and ln % 8 == 0 and rid == i
        key = b[s + 16: s + 48].split(b"\x00")[0]
        assert 8 <= len(key) <= 32
