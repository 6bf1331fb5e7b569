"""The multithreaded CPU baseline (paper variant ii) computes the same results as the oracle."""
import numpy as np

import baselines
import gen
import oracle


def test_mt_baseline_matches_oracle():
    buf, off = gen.grep_records(max_bytes=4 << 20)
    assert np.array_equal(baselines.grep(buf, off), oracle.grep(buf, off))
    g = gen.groupby(n=300_001, zipf=True)
    c, q, a = baselines.groupby(g, 300_001)
    wc, wq, wa = oracle.groupby(g, 300_001, 16, 4096)
    assert np.array_equal(c, wc) and np.array_equal(q, wq)
    np.testing.assert_allclose(a, wa, rtol=1e-9)
    x = gen.points(n=50_000)
    c, s = baselines.kmeans(x, x[:64])
    kc, ks, _, _ = oracle.kmeans(x, x[:64])
    assert np.array_equal(c, kc)
    np.testing.assert_allclose(s, ks, rtol=1e-9)
    assert baselines.threads() >= 1


def test_mt_partition_and_kmer_match_oracle():
    kv = gen.kv(n=200_003)
    for B in (1024, 1):
        boff, out = baselines.partition(kv, B)
        wboff, wout = oracle.partition(kv, B)
        assert np.array_equal(boff, wboff) and np.array_equal(out, wout)
    d = gen.dna(n=5000, genome_len=1 << 14, err_pm=3, n_pm=3)
    km, ct = baselines.kmer(d, 5000)
    okm, oct_ = oracle.kmer(d, 5000)
    assert np.array_equal(km, okm) and np.array_equal(ct, oct_)


def test_mt_wordcount_matches_oracle():
    adv = b"  a\tb\r\n\x00\xff  \x0b\x0cab" + b"ab" + b"" + b"x y  x"
    adv_off = np.array([0, 17, 19, 19], np.uint64)   # records: adversarial, "ab", empty, "x y  x"
    cases = (gen.text(cap_bytes=3 << 20), gen.text(cap_recs=1), (np.zeros(0, np.uint8), np.zeros(0, np.uint64)),
             (np.frombuffer(adv, np.uint8).copy(), adv_off))
    for buf, off in cases:
        b = buf.tobytes()
        wo, wl, wc = baselines.wordcount(buf, off)
        got = sorted((b[int(o): int(o) + int(l)], int(c)) for o, l, c in zip(wo, wl, wc))
        assert got == oracle.wc(buf, off)
