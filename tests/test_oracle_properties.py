"""Property-based pins of the oracle (hypothesis): on arbitrary small inputs — shrunk to minimal
counterexamples on failure — every oracle function equals an independent brute-force formulation
of the definition it follows. None of these formulations
share code with oracle/oracle.c or with the CUDA path."""
import struct
from collections import Counter
from fractions import Fraction

import numpy as np
from hypothesis import HealthCheck, given, settings
from hypothesis import strategies as st

import oracle
from _pins import fmaf_exact, mix64, sub_f32, words_of_record

SETTINGS = dict(max_examples=150, deadline=None, suppress_health_check=[HealthCheck.too_slow])

# bytes biased towards delimiters, NUL, high bytes and a tiny alphabet, so words repeat
BYTE = st.sampled_from(list(b" \t\n\r\x0b\x0c\x00\x80\xffab") + [ord("c")])
RECORD = st.lists(BYTE, max_size=24).map(bytes)


def _records(recs):
    buf = b"".join(recs)
    off = np.cumsum([0] + [len(r) for r in recs[:-1]]).astype(np.uint64) if recs else np.zeros(0, np.uint64)
    return buf, off


@settings(**SETTINGS)
@given(st.lists(RECORD, max_size=12))
def test_wc_equals_split_per_record(recs):
    """O1: the multiset of maximal non-isspace runs per record, sorted by memcmp order."""
    buf, off = _records(recs)
    c = Counter()
    for r in recs:
        c.update(words_of_record(r))
    assert oracle.wc(buf, off) == sorted(c.items())


KEYBYTE = st.sampled_from(list(b"bigkx\x00"))


@settings(**SETTINGS)
@given(st.lists(st.tuples(st.lists(KEYBYTE, min_size=32, max_size=32).map(bytes),
                          st.integers(0, 40)), max_size=10),
       st.lists(st.sampled_from(list(b"bigkx")), max_size=6).map(bytes), st.integers(0, 1000))
def test_grep_equals_substring_of_strnlen_key(rows, pat, first):
    """O2: record i matches iff pat occurs in key[:strnlen(key, 32)] (key at +16); ascending
    indices offset by `first`."""
    recs = [struct.pack("<IIQ", 48 + pl, 0, i) + key + b"p" * pl for i, (key, pl) in enumerate(rows)]
    buf, off = _records(recs)
    want = []
    for i, (key, _) in enumerate(rows):
        kl = key.find(b"\x00")
        kl = 32 if kl < 0 else kl
        if pat in key[:kl]:
            want.append(first + i)
    assert oracle.grep(np.frombuffer(buf, np.uint8) if buf else b"", off, pat, first=first).tolist() == want


@settings(**SETTINGS)
@given(st.lists(st.integers(0, 2**64 - 1), max_size=40), st.sampled_from([1, 2, 4, 1024]))
def test_partition_equals_stable_sort_by_bucket(keys, B):
    """O4: records ordered by (mix64(key) >> (64 - log2 B), original index); offsets per bucket."""
    kv = np.array([[k, i] for i, k in enumerate(keys)], np.uint64).reshape(-1, 2)
    bits = B.bit_length() - 1
    bk = [(mix64(k) >> (64 - bits)) if bits else 0 for k in keys]
    order = sorted(range(len(keys)), key=lambda i: (bk[i], i))
    boff, out = oracle.partition(kv, B)
    assert out.tolist() == [[keys[i], i] for i in order]
    assert boff.tolist() == [sum(1 for b in bk if b < x) for x in range(B + 1)]


@settings(**SETTINGS)
@given(st.lists(st.tuples(st.integers(0, 7), st.integers(0, 2**32 - 1), st.integers(0, 10**5 - 1)), max_size=40),
       st.sampled_from([16, 64]))
def test_groupby_equals_per_key_sums(rows, stride):
    """O5: dense per-key count, qty (mod 2^64) and amount (cents / 100, summed in record order)."""
    buf = b"".join(struct.pack("<IId", k, q, c / 100.0) + b"\xee" * (stride - 16) for k, q, c in rows)
    count, qty, amt = oracle.groupby(np.frombuffer(buf, np.uint8) if buf else b"", len(rows), stride, 8)
    for g in range(8):
        sel = [r for r in rows if r[0] == g]
        assert int(count[g]) == len(sel)
        assert int(qty[g]) == sum(q for _, q, _ in sel) % 2**64
        exact = sum(c for _, _, c in sel) / 100.0
        assert abs(float(amt[g]) - exact) <= 1e-12 * max(1.0, exact)


# fp32 coordinates, zero or of magnitude in [2^-10, 64]: every difference and square stays in the
# normal fp32 range, where _pins.round_f32 (exact rational -> nearest fp32) applies
F32 = st.one_of(st.just(0.0), st.floats(2.0 ** -10, 64, width=32), st.floats(-64, -(2.0 ** -10), width=32),
                st.integers(-64, 64).map(float))


@settings(**SETTINGS)
@given(st.lists(st.lists(F32, min_size=16, max_size=16), max_size=12),
       st.lists(st.lists(F32, min_size=16, max_size=16), min_size=1, max_size=5), st.integers(0, 100))
def test_kmeans_equals_sequential_fp32_argmin(points, cents, first):
    """O3: fp32 distance acc = fmaf(x_j - mu_j, x_j - mu_j, acc) for j ascending, each operation
    rounded once to fp32 in exact rational arithmetic, argmin with ties to the lowest k (integer
    coordinates make ties frequent); counts, fp64 sums and the mix64 checksum."""
    x = np.array(points, np.float32).reshape(-1, 16)
    mu = np.array(cents, np.float32).reshape(-1, 16)
    count, s, chk, cid = oracle.kmeans(x, mu, first=first, want_cid=True)
    K = len(mu)
    wc_ = [0] * K
    ws = np.zeros((K, 16))
    wchk = 0
    for i, p in enumerate(x):
        best, bestd = 0, None
        for k in range(K):
            acc = Fraction(0)
            for j in range(16):
                t = sub_f32(Fraction(float(p[j])), Fraction(float(mu[k, j])))
                acc = fmaf_exact(t, t, acc)
            if bestd is None or acc < bestd:
                best, bestd = k, acc
        assert cid[i] == best
        wc_[best] += 1
        ws[best] += p.astype(np.float64)
        wchk = (wchk + mix64(((first + i) << 8) ^ best)) % 2**64
    assert count.tolist() == wc_ and chk == wchk
    np.testing.assert_allclose(s, ws, rtol=1e-12, atol=1e-9)
