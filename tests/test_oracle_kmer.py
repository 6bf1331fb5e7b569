"""Pins for oracle O6 (k-mer counting, NEXT f4; DNA assembly P:955-963, Table I)."""
from collections import Counter

import numpy as np
import pytest

import gen
import oracle

CODE = {"A": 0, "C": 1, "G": 2, "T": 3}


def brute(buf: np.ndarray, n: int, k: int):
    """Independent formulation: slice strings, skip windows containing non-ACGT, base-4 int()."""
    c = Counter()
    b = buf.tobytes()
    for r in range(n):
        s = b[r * 256 + 16: r * 256 + 112].decode("ascii")
        for j in range(0, 96 - k + 1):
            w = s[j: j + k]
            if set(w) <= set("ACGT"):
                c[int(w.translate(str.maketrans("ACGT", "0123")), 4)] += 1
    keys = sorted(c)
    return np.array(keys, np.uint64), np.array([c[x] for x in keys], np.uint64)


@pytest.mark.parametrize("k", [1, 5, 21, 31])
def test_kmer_vs_brute_force(k):
    buf = gen.dna(n=300, genome_len=5000, err_pm=5, n_pm=10)
    km, ct = oracle.kmer(buf, 300, k)
    bk_, bc = brute(buf, 300, k)
    assert np.array_equal(km, bk_) and np.array_equal(ct, bc)


def test_kmer_special_cases():
    rec = bytearray(256)
    rec[16:112] = b"A" * 96
    buf = np.frombuffer(bytes(rec), np.uint8)
    km, ct = oracle.kmer(buf, 1, 31)
    assert list(km) == [0] and list(ct) == [96 - 31 + 1]         # AAAA...: one k-mer, 66 times
    rec[16 + 40] = ord("N")                                      # an N breaks every window over it
    km, ct = oracle.kmer(np.frombuffer(bytes(rec), np.uint8), 1, 31)
    assert list(ct) == [(40 - 31 + 1) + (96 - 41 - 31 + 1)]
    rec[16:112] = b"ACGT" * 24
    km, ct = oracle.kmer(np.frombuffer(bytes(rec), np.uint8), 1, 4)
    assert list(km) == sorted(int(w, 4) for w in ("0123", "1230", "2301", "3012"))
    assert oracle.kmer(np.zeros(0, np.uint8), 0, 31)[0].size == 0


def test_kmer_invariants():
    buf = gen.dna(n=2000, genome_len=1 << 16, err_pm=1, n_pm=2)
    for k in (11, 31):
        km, ct = oracle.kmer(buf, 2000, k)
        b = buf.tobytes()
        windows = 0
        for r in range(2000):
            s = b[r * 256 + 16: r * 256 + 112]
            bad = [i for i, ch in enumerate(s) if ch not in b"ACGT"]
            windows += sum(1 for j in range(96 - k + 1) if not any(j <= x < j + k for x in bad))
        assert int(ct.sum()) == windows                      # every valid window counted once
        assert np.all(np.diff(km.astype(np.int64)) > 0)     # distinct, ascending
        assert int(km.max()) < 4 ** k


def test_window_helper_of_the_bench_scale_test_matches_oracle():
    """tests/test_gpu_kmer.py recounts sampled k-mers with a numpy helper; pin it to O6 here."""
    from test_gpu_kmer import _windows
    n, k = 300, 13
    buf = gen.dna(n=n, genome_len=1 << 12, err_pm=5, n_pm=20)
    wk, wc = oracle.kmer(buf, n, k)
    val, valid = _windows(buf.reshape(n, 256)[:, 16:112], k)
    u, c = np.unique(val[valid], return_counts=True)
    assert np.array_equal(u, wk) and np.array_equal(c.astype(np.uint64), wc)
