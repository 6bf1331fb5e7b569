"""GPU edge cases of every built-in kernel in every gather mode: the empty data set, one record,
a warp's worth plus one (a ragged tile), and a few hundred records (a ragged lane tail), each
compared with the oracle on the same seeded input (bit-exact; fp64 sums within 1e-5 relative)."""
import numpy as np
import pytest

import gen
import oracle
from paper_conf_ipps_mokhtaris14_b200 import bk

pytestmark = pytest.mark.gpu

MIB = 1 << 20
MODES = ["dense", "zc", "cpu", "hybrid"]
SIZES = [0, 1, 33, 517]


def _ctx(mode, **kw):
    return bk.Context(window_bytes=1 * MIB, gather_mode=mode, **kw)


@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("n", SIZES)
def test_wordcount_and_grep_edges(mode, n):
    if n:
        buf, off = gen.text(cap_recs=n)
        off = off[:n]
    else:
        buf, off = np.zeros(0, np.uint8), np.zeros(0, np.uint64)
    with _ctx(mode) as ctx:
        ctx.register(buf, off)
        o, l, c = ctx.wordcount(cap=1 << 14)
        b = buf.tobytes()
        assert sorted((b[int(x): int(x) + int(y)], int(z)) for x, y, z in zip(o, l, c)) == oracle.wc(buf, off)
    if n:
        gb, goff = gen.grep_records(n=n)
    else:
        gb, goff = np.zeros(0, np.uint8), np.zeros(0, np.uint64)
    with _ctx(mode) as ctx:
        ctx.register(gb, goff)
        for pat in (b"bigk", b"", b"a"):
            got = ctx.grep(pat, cap=max(len(goff), 1))
            assert np.array_equal(got, oracle.grep(gb, goff, pat)), pat


@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("n", SIZES)
def test_fixed_record_kernels_edges(mode, n):
    # group-by (16-B records)
    g = gen.groupby(n=n) if n else np.zeros(0, np.uint8)
    with _ctx(mode, record_size=16) as ctx:
        ctx.register(g, None, n_records=n)
        c, q, a = ctx.groupby(4096)
    wc_, wq, wa = oracle.groupby(g, n, 16, 4096)
    assert np.array_equal(c, wc_) and np.array_equal(q, wq)
    np.testing.assert_allclose(a, wa, rtol=1e-5, atol=0)
    # k-means (64-B points), centroids from elsewhere so n < K is legal
    x = gen.points(n=n) if n else np.zeros((0, 16), np.float32)
    mu = gen.points(first=1 << 30, n=64)
    with _ctx(mode, record_size=64) as ctx:
        ctx.register(x.view(np.uint8).reshape(-1), None, n_records=n)
        cid = np.full(max(n, 1), -1, np.int32)
        kc, ks, kchk = ctx.kmeans(mu, cid=cid)
    oc, os_, ochk, ocid = oracle.kmeans(x, mu, want_cid=True)
    assert np.array_equal(kc, oc) and kchk == ochk
    assert np.array_equal(cid[:n], ocid)
    np.testing.assert_allclose(ks, os_, rtol=1e-5, atol=0)
    # k-mers (256-B read records)
    d = gen.dna(n=n) if n else np.zeros(0, np.uint8)
    with _ctx(mode, record_size=256) as ctx:
        ctx.register(d, None, n_records=n)
        km, ct, tot = ctx.kmer(k=31, cap=1 << 16)
    okm, oct_ = oracle.kmer(d, n, k=31)
    order = np.argsort(km)
    assert np.array_equal(km[order], okm) and np.array_equal(ct[order], oct_)
    assert tot == int(oct_.sum())


@pytest.mark.parametrize("mode", ["dense", "zc", "cpu"])
@pytest.mark.parametrize("n", SIZES)
def test_partition_edges(mode, n):
    kv = gen.kv(n=n) if n else np.zeros((0, 2), np.uint64)
    with _ctx(mode, record_size=16) as ctx:
        ctx.register(kv.view(np.uint8).reshape(-1), None, n_records=n)
        out, cc, bc = ctx.partition(64)
    boff, want = oracle.partition(kv, 64)
    assert np.array_equal(np.concatenate([[0], np.cumsum(bc)]).astype(np.uint64), boff)
    # chunk-major runs -> bucket-major order (stable within a bucket)
    got = np.empty_like(want)
    pos = boff[:-1].astype(np.int64).copy()
    src = 0
    for row in cc:
        for b, m in enumerate(row):
            m = int(m)
            got[pos[b]: pos[b] + m] = out[src: src + m]
            pos[b] += m
            src += m
    assert src == n and np.array_equal(got, want)
