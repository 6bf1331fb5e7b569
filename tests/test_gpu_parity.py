"""GPU parity: the CUDA path through the C ABI vs the CPU oracle on the same seeded inputs.

Bit-exact for counts, indices, words and staged bytes; fp64 sums within 1e-5 relative
(north_star). Sizes span many chunks, several tiles per chunk and ragged tails.
"""
import struct

import numpy as np
import pytest

import gen
import oracle
from paper_conf_ipps_mokhtaris14_b200 import bk

pytestmark = pytest.mark.gpu

MIB = 1 << 20


def wc_multiset_gpu(buf: np.ndarray, off_, ln, cnt):
    b = buf.tobytes()
    return sorted((b[int(o): int(o) + int(l)], int(c)) for o, l, c in zip(off_, ln, cnt))


# ------------------------------------------------------------------ layout (stages 1-2)
LAYOUT_CASES = [
    # name, extents, fixed record size
    ("wc_text", None, 0),
    ("grep_key", [(16, 32)], 0),
    ("sparse64", [(0, 16)], 64),
    ("kmeans64", None, 64),
    ("dup_extents", [(8, 4), (0, 12), (8, 4)], 16),
    ("grep_multi", [(16, 8), (40, 8)], 0),
]


def layout_data(name):
    if name == "wc_text":
        buf, off = gen.text(cap_bytes=300_000)
        return buf, off, 0
    if name in ("grep_key", "grep_multi"):
        buf, off = gen.grep_records(n=5000)
        return buf, off, 0
    if name == "sparse64":
        return gen.groupby(n=7001, stride=64), None, 64
    if name == "kmeans64":
        return gen.points(n=3001).view(np.uint8).reshape(-1), None, 64
    return gen.groupby(n=4099, stride=16), None, 16


@pytest.mark.parametrize("name,extents,rs", LAYOUT_CASES)
@pytest.mark.parametrize("mode", ["zc", "dense", "cpu"])
@pytest.mark.parametrize("lanes", [32, 160])
def test_layout_dump_matches_oracle(name, extents, rs, mode, lanes):
    buf, off, rs = layout_data(name)
    n = len(off) if off is not None else len(buf) // rs
    chunk = 12_000
    with bk.Context(window_bytes=8 * MIB, n_slots=2, gather_mode=mode, chunk_bytes=chunk, lanes=lanes,
                    record_size=rs) as ctx:
        ctx.register(buf, off, n_records=n)
        # the plan budget counts accessed bytes in zc mode, whole records in dense mode
        plan_ext = None if mode == "dense" else extents
        bounds = oracle.plan_chunks(off, n, len(buf), rs, plan_ext, chunk)
        first = ctx.layout_dump(0, extents)
        assert first["n_chunks"] == len(bounds) - 1 >= 3
        for c in sorted({0, 1, len(bounds) // 2, len(bounds) - 2}):
            got = ctx.layout_dump(c, extents)
            assert (got["lo"], got["hi"]) == (int(bounds[c]), int(bounds[c + 1]))
            stage, lf, ln, lb = oracle.layout(buf, off, n, len(buf), rs, extents, got["lo"], got["hi"], got["lanes"])
            assert np.array_equal(got["lane_first"], lf)
            assert np.array_equal(got["lane_nrec"], ln)
            assert np.array_equal(got["lane_bytes"], lb)
            assert got["stage"].tobytes() == stage.tobytes()


# ------------------------------------------------------------------ C1 word count
@pytest.mark.parametrize("mode", ["dense", "zc", "cpu", "hybrid", "fused"])
@pytest.mark.parametrize("window,slots", [(256 * 1024, 2), (1 * MIB, 4), (8 * MIB, 3)])
def test_wordcount_small(mode, window, slots):
    buf, off = gen.text(cap_bytes=2 * MIB)
    want = oracle.wc(buf, off)
    with bk.Context(window_bytes=window, n_slots=slots, gather_mode=mode) as ctx:
        ctx.register(buf, off)
        got = wc_multiset_gpu(buf, *ctx.wordcount(cap=1 << 18))
        st = ctx.stats()
        assert st["n_chunks"] >= 2
        if mode == "fused":   # one persistent launch; its shared-memory ring stays inside the window
            assert st["gather_mode"] == bk.BK_GATHER_FUSED and st["n_units"] == st["n_chunks"]
            assert st["fused_ring_slots"] >= 2 and 1 <= st["fused_loaders"] < st["fused_grid"]
            assert st["fused_ring_slots"] * (st["unit_bytes"] * 3 // 2) <= window   # ring inside the window
            assert st["bytes_accessed"] == len(buf) and st["bytes_meta"] == 8 * len(off)
    assert got == want


@pytest.mark.parametrize("profile", [False, True])
def test_wordcount_fused_repeat_and_profile(profile):
    """The fused kernel replayed from its graph gives the same table every run; profiled runs
    report the in-kernel wait / compute shares."""
    buf, off = gen.text(cap_bytes=3 * MIB)
    want = oracle.wc(buf, off)
    with bk.Context(window_bytes=2 * MIB, profile=profile) as ctx:
        ctx.register(buf, off)
        for _ in range(3):
            assert wc_multiset_gpu(buf, *ctx.wordcount(cap=1 << 18)) == want
        st = ctx.stats()
    assert st["gather_mode"] == bk.BK_GATHER_FUSED
    if profile:
        assert 0 <= st["fused_wait_frac"] < 1 and 0 < st["fused_compute_frac"] < 1
        assert 0 <= st["fused_loader_wait_frac"] < 1 and st["ms_zc"] > 0


def adversarial_text():
    """Mixed delimiter runs, empty records, bytes 0x00 / >= 0x80 as word bytes, a last record
    without a newline, a 300-byte word (SURVEY §8(c) adversarial catalogue)."""
    recs = [b"  a\tb\r\n", b"", b"", b"\x00\x80 z", b"ab", b"cd", b"tail without newline", b" ", b"x" * 300,
            b"dup dup\n"] * 37
    buf = np.frombuffer(b"".join(recs), np.uint8)
    off = np.cumsum([0] + [len(r) for r in recs[:-1]]).astype(np.uint64)
    return buf, off


def test_wordcount_adversarial():
    buf, off = adversarial_text()
    want = oracle.wc(buf, off)
    for mode in ("zc", "dense", "cpu", "hybrid"):
        with bk.Context(window_bytes=64 * 1024, n_slots=2, gather_mode=mode, chunk_bytes=1500, lanes=32) as ctx:
            ctx.register(buf, off)
            assert wc_multiset_gpu(buf, *ctx.wordcount(cap=4096)) == want
    # the fused single launch: many small units (window 64 KiB -> few CTAs, 2 KiB units) and the default
    for window in (64 * 1024, 8 * MIB):
        with bk.Context(window_bytes=window, gather_mode="fused") as ctx:
            ctx.register(buf, off)
            assert wc_multiset_gpu(buf, *ctx.wordcount(cap=4096)) == want
            assert ctx.stats()["gather_mode"] == bk.BK_GATHER_FUSED


def test_wordcount_full_c1_config():
    """configs[0]: 64 MiB text, 8 MiB window, 1 GPU — whole result bit-exact vs the oracle."""
    buf, off = gen.text(cap_bytes=64 * MIB)
    want = oracle.wc(buf, off)
    with bk.Context(window_bytes=8 * MIB) as ctx:
        ctx.register(buf, off)
        got = wc_multiset_gpu(buf, *ctx.wordcount(cap=1 << 20))
        st = ctx.stats()
    assert got == want
    assert st["bytes_accessed"] == len(buf)        # I3: every byte accessed once
    assert st["n_chunks"] >= 8                      # out-of-core: data > window
    assert st["gather_mode"] == bk.BK_GATHER_FUSED  # AUTO: the single persistent launch


# ------------------------------------------------------------------ C2 grep
def grep_rec(key: bytes, payload: bytes = b"") -> bytes:
    k = key[:32].ljust(32, b"\x00")
    return struct.pack("<IIQ", 48 + len(payload), 0, 0) + k + payload


def test_grep_adversarial():
    recs = [grep_rec(b"bigkxxxx"), grep_rec(b"xxxxbigk"), grep_rec(b"a" * 28 + b"bigk"), grep_rec(b"big\x00k"),
            grep_rec(b"bi"), grep_rec(b"xbigkx", b"bigkbigk" + b"q" * 7), grep_rec(b""), grep_rec(b"q" * 32, b"z")] * 53
    buf = np.frombuffer(b"".join(recs), np.uint8)
    off = np.cumsum([0] + [len(r) for r in recs[:-1]]).astype(np.uint64)
    for pat in (b"bigk", b"", b"a", b"q" * 32, b"aaaaaaaaaaaabigk", b"x" * 33):
        if len(pat) > 32:
            with bk.Context(window_bytes=1 * MIB) as ctx:
                ctx.register(buf, off)
                with pytest.raises(bk.BkError):
                    ctx.grep(pat)
            continue
        want = oracle.grep(buf, off, pat)
        for mode in ("zc", "dense", "cpu", "hybrid"):
            with bk.Context(window_bytes=256 * 1024, n_slots=2, gather_mode=mode, chunk_bytes=2048, lanes=64) as ctx:
                ctx.register(buf, off)
                got = ctx.grep(pat, cap=len(off))
            assert np.array_equal(got, want), (pat, mode)


@pytest.mark.parametrize("mode", ["zc", "dense", "cpu", "hybrid"])
def test_grep_medium(mode):
    buf, off = gen.grep_records(max_bytes=64 * MIB)
    want = oracle.grep(buf, off, b"bigk", first=1000)
    with bk.Context(window_bytes=16 * MIB, gather_mode=mode) as ctx:
        ctx.register(buf, off)
        got = ctx.grep(b"bigk", first_index=1000, cap=len(off))
        st = ctx.stats()
    assert np.array_equal(got, want)
    assert st["n_chunks"] >= 8
    if mode == "zc":
        assert st["bytes_accessed"] == 32 * len(off) == st["bytes_h2d"]   # I3: only the key bytes
    if mode == "cpu":
        assert st["n_chunks_cpu"] == st["n_chunks"] and st["bytes_meta"] == 0
        assert 32 * len(off) <= st["bytes_h2d"] <= 32 * len(off) * 1.05  # packed keys + tile padding
    if mode == "hybrid":
        assert 0 < st["n_chunks_cpu"] < st["n_chunks"]


@pytest.mark.parametrize("mode", ["zc", "cpu"])
def test_grep_every_pattern_length(mode):
    """The SWAR matcher at every pattern length 1..32: each pattern is cut from a real key (so it
    matches somewhere), from its start, middle or end; indices equal the oracle's."""
    buf, off = gen.grep_records(n=30_000)
    b = buf.tobytes()
    rng = np.random.default_rng(7)
    with bk.Context(window_bytes=4 * MIB, gather_mode=mode) as ctx:
        ctx.register(buf, off)
        for L in range(1, 33):
            for _ in range(2):
                r = int(rng.integers(len(off)))
                key = b[int(off[r]) + 16: int(off[r]) + 48].split(b"\0")[0]
                if len(key) < L:
                    key = (key * 8)[:32]   # repeated key bytes: still a plausible pattern, maybe no match
                s0 = int(rng.integers(0, len(key) - L + 1))
                pat = key[s0: s0 + L]
                got = ctx.grep(pat, cap=len(off))
                assert np.array_equal(got, oracle.grep(buf, off, pat)), (L, pat)


@pytest.mark.parametrize("lane_bytes", [1024, 1056, 4096])
def test_grep_long_lanes(lane_bytes):
    """Lanes of 32, 33 and 128 keys: k_grep_count keeps a 32-record match mask per lane; longer
    lanes are re-tested from the staged keys by k_grep_write. Same indices as the oracle."""
    buf, off = gen.grep_records(n=60_000)
    for pat in (b"bigk", b"", b"a"):
        want = oracle.grep(buf, off, pat, first=5)
        for mode in ("zc", "hybrid"):
            with bk.Context(window_bytes=8 * MIB, gather_mode=mode, lane_bytes=lane_bytes) as ctx:
                ctx.register(buf, off)
                got = ctx.grep(pat, first_index=5, cap=len(off))
            assert np.array_equal(got, want), (pat, mode, lane_bytes)


def test_grep_capacity_error():
    buf, off = gen.grep_records(n=20000)
    with bk.Context(window_bytes=4 * MIB) as ctx:
        ctx.register(buf, off)
        with pytest.raises(bk.BkError) as e:
            ctx.grep(b"", cap=100)
        assert e.value.status == bk.BK_E_CAPACITY


def test_grep_full_c2_config():
    """configs[1] in bench.py's launch configuration: 16 GiB, 2 GiB window, zc gather.
    The oracle computes the whole answer (single-threaded C, ~10 s)."""
    buf, off = gen.grep_records(max_bytes=16 << 30)
    with bk.Context(window_bytes=2 << 30) as ctx:
        ctx.register(buf, off)
        got = ctx.grep(b"bigk", cap=len(off) // 50)
        st = ctx.stats()
    want = oracle.grep(buf, off, b"bigk")
    assert np.array_equal(got, want)
    assert st["n_chunks"] >= 16 and st["bytes_accessed"] == 32 * len(off)


# ------------------------------------------------------------------ C5 group-by
@pytest.mark.parametrize("stride,zipf,mode", [(16, False, "dense"), (16, True, "zc"), (64, False, "zc"),
                                              (64, True, "dense"), (64, False, "cpu"), (16, True, "hybrid")])
def test_groupby(stride, zipf, mode):
    n = 3_000_001
    buf = gen.groupby(n=n, stride=stride, zipf=zipf)
    wc_, wq, wa = oracle.groupby(buf, n, stride, 4096)
    with bk.Context(window_bytes=16 * MIB, gather_mode=mode, record_size=stride) as ctx:
        ctx.register(buf, None, n_records=n)
        c, q, a = ctx.groupby(4096)
        assert ctx.stats()["n_chunks"] >= 4
    assert np.array_equal(c, wc_) and np.array_equal(q, wq)
    np.testing.assert_allclose(a, wa, rtol=1e-5, atol=0)


@pytest.mark.parametrize("G,mode", [(8192, "dense"), (1, "dense"), (8192, "zc"), (4097, "cpu")])
def test_groupby_group_counts(G, mode):
    """Table sizes at the edges: G = 8192 halves the TMA pieces (4 rows) to fit the shared table,
    G = 1 sends every record to one slot; both load paths (TMA in dense/cpu, plain loads in zc)."""
    n = 1_000_003
    buf = gen.groupby(n=n, G=G)
    wc_, wq, wa = oracle.groupby(buf, n, 16, G)
    with bk.Context(window_bytes=8 * MIB, gather_mode=mode, record_size=16) as ctx:
        ctx.register(buf, None, n_records=n)
        c, q, a = ctx.groupby(G)
    assert np.array_equal(c, wc_) and np.array_equal(q, wq)
    np.testing.assert_allclose(a, wa, rtol=1e-5, atol=0)


def test_groupby_key_out_of_range():
    buf = gen.groupby(n=1000, G=4096)
    with bk.Context(window_bytes=1 * MIB, record_size=16) as ctx:
        ctx.register(buf, None, n_records=1000)
        with pytest.raises(bk.BkError) as e:
            ctx.groupby(G=100)
        assert e.value.status == bk.BK_E_INVAL


# ------------------------------------------------------------------ C3 k-means
@pytest.mark.parametrize("mode,K", [("dense", 64), ("zc", 64), ("dense", 7), ("cpu", 64), ("hybrid", 33),
                                    ("dense", 1), ("cpu", 256), ("zc", 255)])
def test_kmeans(mode, K):
    n = 400_003
    x = gen.points(n=n)
    mu = x[:K].copy()
    wc_, ws, wchk, _ = oracle.kmeans(x, mu, first=5)
    with bk.Context(window_bytes=8 * MIB, gather_mode=mode, record_size=64) as ctx:
        ctx.register(x.view(np.uint8).reshape(-1), None, n_records=n)
        c, s, chk = ctx.kmeans(mu, first_index=5)
    assert np.array_equal(c, wc_) and chk == wchk
    # |gpu - ref| <= 1e-5 * sum |x| (data are positive, so this is relative)
    np.testing.assert_allclose(s, ws, rtol=1e-5, atol=0)


# ------------------------------------------------------------------ C4 partition
def global_from_runs(out, cc):
    """Stable global partition from chunk-major bucket-sorted runs: bucket b = chunk 0's run of b,
    then chunk 1's, ... (chunks ascend in record order)."""
    C, B = cc.shape
    starts = np.zeros((C, B), np.int64)
    lo = 0
    for c in range(C):
        starts[c] = lo + np.concatenate([[0], np.cumsum(cc[c].astype(np.int64))[:-1]])
        lo += int(cc[c].sum())
    parts = [out[starts[c, b]: starts[c, b] + int(cc[c, b])] for b in range(B) for c in range(C) if cc[c, b]]
    return np.concatenate(parts) if parts else out[:0]


@pytest.mark.parametrize("B,mode,n", [(1024, "dense", 1_000_003), (1024, "zc", 300_001), (1, "dense", 100_000),
                                      (4096, "cpu", 200_000), (16, "hybrid", 500_000)])
def test_partition(B, mode, n):
    kv = gen.kv(n=n)
    wboff, wout = oracle.partition(kv, B)
    with bk.Context(window_bytes=8 * MIB, gather_mode=mode, record_size=16) as ctx:
        ctx.register(kv.view(np.uint8).reshape(-1), None, n_records=n)
        out, cc, bc = ctx.partition(B)
        st = ctx.stats()
    assert cc.shape[0] == st["n_chunks"] >= 2
    assert np.array_equal(np.concatenate([[0], np.cumsum(bc)]).astype(np.uint64), wboff)
    assert np.array_equal(global_from_runs(out, cc), wout)
    assert st["bytes_d2h"] == 16 * n


def test_partition_duplicate_keys_and_errors():
    kv = np.array([[7, i] for i in range(5000)] + [[9, i] for i in range(5000, 7000)], np.uint64)
    with bk.Context(window_bytes=1 * MIB, record_size=16) as ctx:
        ctx.register(kv.view(np.uint8).reshape(-1), None, n_records=len(kv))
        out, cc, bc = ctx.partition(1024)
        assert np.array_equal(global_from_runs(out, cc), oracle.partition(kv, 1024)[1])
        with pytest.raises(bk.BkError):
            ctx.partition(1000)
        with pytest.raises(bk.BkError) as e:
            ctx.partition(1024, chunk_cap=1)
        assert e.value.status == bk.BK_E_CAPACITY


# ------------------------------------------------------------------ the double-buffering baseline
@pytest.mark.parametrize("sbuf", [False, True])
def test_dbuf_baseline_wordcount_matches_oracle(sbuf):
    """The word-count double- (and single-) buffering baseline: the same word multiset (I2), also
    on the adversarial text (empty records, delimiter runs, high bytes)."""
    buf, off = gen.text(cap_bytes=3 * MIB)
    for b, o in ((buf, off), adversarial_text()):
        want = oracle.wc(b, o)
        with bk.Context(window_bytes=512 * 1024, baseline_dbuf=not sbuf, baseline_sbuf=sbuf) as ctx:
            ctx.register(b, o)
            assert wc_multiset_gpu(b, *ctx.wordcount(cap=1 << 17)) == want


@pytest.mark.parametrize("sbuf", [False, True])
def test_dbuf_baseline_kmeans_matches_oracle(sbuf):
    """The k-means double- (and single-) buffering baseline: same counts, checksum and sums (I2)."""
    n, K = 300_007, 64
    x = gen.points(n=n)
    mu = x[:K].copy()
    wc_, ws, wchk, _ = oracle.kmeans(x, mu, first=3)
    with bk.Context(window_bytes=4 * MIB, baseline_dbuf=not sbuf, baseline_sbuf=sbuf, record_size=64) as ctx:
        ctx.register(x.view(np.uint8).reshape(-1), None, n_records=n)
        c, s, chk = ctx.kmeans(mu, first_index=3)
        assert ctx.stats()["n_chunks"] >= 4
        with pytest.raises(bk.BkError):   # no cid write-back in the baseline
            ctx.kmeans(mu, cid=np.empty(n, np.int32))
    assert np.array_equal(c, wc_) and chk == wchk
    np.testing.assert_allclose(s, ws, rtol=1e-5, atol=0)


def test_dbuf_baseline_grep_and_groupby_match_oracle():
    """BK_FLAG_BASELINE_DBUF (the paper's variant iv) must give the same results (I2)."""
    buf, off = gen.grep_records(max_bytes=24 * MIB)
    want = oracle.grep(buf, off, b"bigk", first=7)
    with bk.Context(window_bytes=4 * MIB, baseline_dbuf=True) as ctx:
        ctx.register(buf, off)
        got = ctx.grep(b"bigk", first_index=7, cap=len(off))
        assert ctx.stats()["n_chunks"] >= 8
    assert np.array_equal(got, want)
    n = 2_000_003
    g = gen.groupby(n=n, zipf=True)
    wc_, wq, wa = oracle.groupby(g, n, 16, 4096)
    with bk.Context(window_bytes=4 * MIB, baseline_dbuf=True, record_size=16) as ctx:
        ctx.register(g, None, n_records=n)
        c, q, a = ctx.groupby(4096)
    assert np.array_equal(c, wc_) and np.array_equal(q, wq)
    np.testing.assert_allclose(a, wa, rtol=1e-5, atol=0)


# ------------------------------------------------------------------ f1: k-means cid write-back
@pytest.mark.parametrize("mode", ["dense", "zc", "hybrid"])
def test_kmeans_cid_writeback(mode):
    n = 300_007
    x = gen.points(n=n)
    mu = x[:64].copy()
    wc_, ws, wchk, wcid = oracle.kmeans(x, mu, want_cid=True)
    cid = np.full(n, -1, np.int32)
    with bk.Context(window_bytes=4 * MIB, gather_mode=mode, record_size=64) as ctx:
        ctx.register(x.view(np.uint8).reshape(-1), None, n_records=n)
        c, s, chk = ctx.kmeans(mu, cid=cid)
        assert ctx.stats()["bytes_d2h"] >= 4 * n
        c2, _, _ = ctx.kmeans(mu)   # without write-back on the same context
    assert np.array_equal(cid, wcid) and np.array_equal(c, wc_) and chk == wchk and np.array_equal(c2, wc_)


# ------------------------------------------------------------------ bench-scale sizes (sampled / properties)
def mix64_np(x):
    x = x.astype(np.uint64)
    x ^= x >> np.uint64(30); x *= np.uint64(0xBF58476D1CE4E5B9)
    x ^= x >> np.uint64(27); x *= np.uint64(0x94D049BB133111EB)
    x ^= x >> np.uint64(31)
    return x


@pytest.mark.parametrize("n", [250_000_000, 500_000_000])
def test_kmeans_bench_scale_sampled(n):
    """2.5e8 points (16 GiB, bench.py's default k-means size) and 5e8 (32 GiB, C3's per-GPU share at
    2 GPUs) in bench.py's launch configuration (2 GiB window, AUTO). Checked: every cid the oracle
    computes for 200k sampled points, Sum count = n, count = bincount(cid), the checksum recomputed
    from the written-back cids, and column sums."""
    x = gen.points(n=n)
    mu = gen.points(n=64)
    cid = np.empty(n, np.int32)
    with bk.Context(window_bytes=2 << 30, record_size=64) as ctx:
        ctx.register(x.view(np.uint8).reshape(-1), None, n_records=n)
        c, s, chk = ctx.kmeans(mu, cid=cid)
    rng = np.random.default_rng(5)
    idx = np.sort(rng.choice(n, 200_000, replace=False))
    _, _, _, scid = oracle.kmeans(x[idx], mu, want_cid=True)
    assert np.array_equal(cid[idx], scid)
    assert int(c.sum()) == n and np.array_equal(c, np.bincount(cid, minlength=64).astype(np.uint64))
    i = np.arange(n, dtype=np.uint64)
    assert int(mix64_np((i << np.uint64(8)) ^ cid.astype(np.uint64)).sum(dtype=np.uint64)) == chk
    np.testing.assert_allclose(s.sum(0), x.sum(0, dtype=np.float64), rtol=1e-9)


def test_partition_bench_scale():
    """C4 per-GPU share (64 GiB / 8 GPUs = 8 GiB, 2^29 records), 1024 buckets: whole result bit-exact."""
    n = 1 << 29
    kv = gen.kv(n=n)
    with bk.Context(window_bytes=2 << 30, record_size=16) as ctx:
        ctx.register(kv.view(np.uint8).reshape(-1), None, n_records=n)
        out, cc, bc = ctx.partition(1024)
    del ctx
    wboff, wout = oracle.partition(kv, 1024)
    assert np.array_equal(np.concatenate([[0], np.cumsum(bc)]).astype(np.uint64), wboff)
    assert np.array_equal(global_from_runs(out, cc), wout)
    assert np.array_equal(bk.partition_materialize(out, cc), wout)   # the host bucket-major pass


def test_groupby_bench_scale():
    """C5 at 32 GiB through a 2 GiB window (16x out-of-core), whole result vs the oracle."""
    n = 2 << 30
    g = gen.groupby(n=n)
    with bk.Context(window_bytes=2 << 30, record_size=16) as ctx:
        ctx.register(g, None, n_records=n)
        c, q, a = ctx.groupby(4096)
        assert ctx.stats()["n_chunks"] >= 16
    wc_, wq, wa = oracle.groupby(g, n, 16, 4096)
    assert np.array_equal(c, wc_) and np.array_equal(q, wq)
    np.testing.assert_allclose(a, wa, rtol=1e-5, atol=0)


# ------------------------------------------------------------------ CUDA-graph replay == eager issue
@pytest.mark.parametrize("no_graph", [False, True])
def test_repeated_runs_graph_replay(no_graph):
    """The first run of a static (ZC/DENSE) pipeline is captured as a CUDA graph, later runs replay
    it; results and stats must equal the eager path on every repetition."""
    buf, off = gen.text(cap_bytes=3 * MIB)
    want = oracle.wc(buf, off)
    gb, goff = gen.grep_records(max_bytes=8 * MIB)
    gwant = oracle.grep(gb, goff, b"bigk")
    n = 200_000
    x = gen.points(n=n)
    kc, ks, kchk, kcid = oracle.kmeans(x, x[:64], want_cid=True)
    kv = gen.kv(n=300_000)
    wboff, wout = oracle.partition(kv, 256)
    with bk.Context(window_bytes=1 * MIB, no_graph=no_graph) as ctx:
        ctx.register(buf, off)
        for _ in range(3):
            assert wc_multiset_gpu(buf, *ctx.wordcount(cap=1 << 17)) == want
            st = ctx.stats()
            assert st["bytes_accessed"] == len(buf) and st["n_chunks"] >= 4
    with bk.Context(window_bytes=2 * MIB, gather_mode="zc", no_graph=no_graph) as ctx:
        ctx.register(gb, goff)
        for pat in (b"bigk", b"zz", b"bigk"):
            got = ctx.grep(pat, cap=len(goff))
            assert np.array_equal(got, oracle.grep(gb, goff, pat))
    with bk.Context(window_bytes=2 * MIB, record_size=64, no_graph=no_graph) as ctx:
        ctx.register(x.view(np.uint8).reshape(-1), None, n_records=n)
        for _ in range(2):
            cid = np.full(n, -1, np.int32)
            c, s, chk = ctx.kmeans(x[:64], cid=cid)
            assert np.array_equal(cid, kcid) and chk == kchk and np.array_equal(c, kc)
    with bk.Context(window_bytes=2 * MIB, record_size=16, no_graph=no_graph) as ctx:
        ctx.register(kv.view(np.uint8).reshape(-1), None, n_records=len(kv))
        out = np.empty_like(kv)
        for _ in range(2):
            out[:] = 0
            o, cc, bc = ctx.partition(256, out=out)
            assert np.array_equal(global_from_runs(o, cc), wout)


@pytest.mark.parametrize("mode", ["dense", "zc", "hybrid"])
def test_profiled_runs(mode):
    """BK_FLAG_PROFILE (the bench's stage-breakdown pass) issues eagerly with CUDA events around every
    stage of every chunk, including the write-back D2H copies issued inside the compute enqueue
    (nested intervals): results equal the oracle and the stage accounting is consistent."""
    x = gen.points(n=150_000)
    kc, ks, kchk, kcid = oracle.kmeans(x, x[:64], want_cid=True)
    kv = gen.kv(n=200_000)
    wboff, wout = oracle.partition(kv, 512)
    gb, goff = gen.grep_records(max_bytes=6 * MIB)
    with bk.Context(window_bytes=2 * MIB, record_size=64, gather_mode=mode, profile=True) as ctx:
        ctx.register(x.view(np.uint8).reshape(-1), None, n_records=len(x))
        cid = np.full(len(x), -1, np.int32)
        c, s, chk = ctx.kmeans(x[:64], cid=cid)
        assert np.array_equal(cid, kcid) and chk == kchk and np.array_equal(c, kc)
        st = ctx.stats()
        assert st["n_d2h"] == st["n_chunks"] and st["ms_d2h"] > 0 and st["bytes_d2h"] >= 4 * len(x)
        assert st["ms_compute"] > 0 and 0 < st["ms_xfer_busy"] <= st["ms_device"] * 1.01
    if mode != "hybrid":
        with bk.Context(window_bytes=2 * MIB, record_size=16, gather_mode=mode, profile=True) as ctx:
            ctx.register(kv.view(np.uint8).reshape(-1), None, n_records=len(kv))
            o, cc, bc = ctx.partition(512)
            assert np.array_equal(global_from_runs(o, cc), wout)
            st = ctx.stats()
            assert st["n_d2h"] == st["n_chunks"] >= 4 and st["ms_d2h"] > 0
            assert st["ms_overlap"] <= min(st["ms_xfer_busy"], st["ms_compute_busy"]) + 1e-6
    with bk.Context(window_bytes=2 * MIB, gather_mode=mode, profile=True) as ctx:
        ctx.register(gb, goff)
        assert np.array_equal(ctx.grep(b"bigk", cap=len(goff)), oracle.grep(gb, goff, b"bigk"))
        st = ctx.stats()
        assert st["n_d2h"] == 0 and st["ms_compute"] > 0 and st["ms_xfer_busy"] > 0


def test_reregistration_and_prepinned_data():
    """One context, several data sets in turn (each registration releases the previous pinning and
    drops cached plans / graphs), plus a caller-pinned buffer that libbk must not re-register."""
    import torch
    t1, o1 = gen.text(cap_bytes=2 * MIB)
    gb, goff = gen.grep_records(n=40_000)
    t2, o2 = gen.text(seed=12345, cap_bytes=1 * MIB)
    with bk.Context(window_bytes=1 * MIB) as ctx:
        for _ in range(2):
            ctx.register(t1, o1)
            assert wc_multiset_gpu(t1, *ctx.wordcount(cap=1 << 17)) == oracle.wc(t1, o1)
            ctx.register(gb, goff)
            assert np.array_equal(ctx.grep(b"bigk", cap=len(goff)), oracle.grep(gb, goff, b"bigk"))
            ctx.register(t2, o2)
            assert wc_multiset_gpu(t2, *ctx.wordcount(cap=1 << 17)) == oracle.wc(t2, o2)
        pinned = torch.empty(len(t1), dtype=torch.uint8, pin_memory=True).numpy()
        pinned[:] = t1
        ctx.register(pinned, o1)
        assert wc_multiset_gpu(pinned, *ctx.wordcount(cap=1 << 17)) == oracle.wc(t1, o1)
    # the caller's pinned buffer is still valid (not unregistered by libbk) after bk_destroy
    assert pinned[:16].tobytes() == t1[:16].tobytes()


# ------------------------------------------------------------------ invariants + API errors
def test_invariance_across_window_slots_lanes_modes():
    buf, off = gen.text(cap_bytes=1 * MIB)
    want = oracle.wc(buf, off)
    for window, slots, lanes, mode in [(128 * 1024, 2, 0, "zc"), (300_000, 3, 64, "dense"), (4 * MIB, 8, 0, "zc"),
                                       (4 * MIB, 2, 1024, "dense"), (512 * 1024, 4, 96, "cpu"),
                                       (1 * MIB, 6, 0, "hybrid")]:
        with bk.Context(window_bytes=window, n_slots=slots, lanes=lanes, gather_mode=mode) as ctx:
            ctx.register(buf, off)
            assert wc_multiset_gpu(buf, *ctx.wordcount(cap=1 << 17)) == want, (window, slots, lanes, mode)


def test_api_errors():
    buf, off = gen.text(cap_bytes=100_000)
    with bk.Context(window_bytes=1 * MIB) as ctx:
        with pytest.raises(bk.BkError) as e:
            ctx.wordcount()
        assert e.value.status == bk.BK_E_STATE
        bad = off.copy()
        bad[5], bad[6] = bad[6], bad[5]
        with pytest.raises(bk.BkError) as e:
            ctx.register(buf, bad)
        assert e.value.status == bk.BK_E_INVAL
    with bk.Context(window_bytes=1 * MIB, chunk_bytes=10) as ctx:   # a line is longer than the budget
        ctx.register(buf, off)
        with pytest.raises(bk.BkError) as e:
            ctx.wordcount()
        assert e.value.status == bk.BK_E_RANGE
    with pytest.raises(bk.BkError):
        bk.Context(n_slots=1)
    # empty data set
    with bk.Context(window_bytes=1 * MIB) as ctx:
        ctx.register(np.zeros(0, np.uint8), np.zeros(0, np.uint64))
        o, l, c = ctx.wordcount(cap=16)
        assert len(c) == 0


# ------------------------------------------------------------------ delay injection
@pytest.mark.parametrize("mode", ["zc", "dense", "cpu", "hybrid", "addr"])
def test_results_survive_random_stage_delays(mode):
    """Random spin kernels before every stage on every stream (and host sleeps before CPU
    assembly) reorder the stages' timing; with a 2-slot ring any missing event dependency
    (slot reuse before its compute finished, compute before its gather) corrupts results."""
    buf, off = gen.text(cap_bytes=1 * MIB)
    want = oracle.wc(buf, off)
    gb, goff = gen.grep_records(max_bytes=4 * MIB)
    gwant = oracle.grep(gb, goff, b"bigk")
    kv = gen.kv(n=200_000)
    wboff, wout = oracle.partition(kv, 1024)
    with bk.Context(window_bytes=256 * 1024, n_slots=2, gather_mode=mode, test_delays=True, no_graph=True) as ctx:
        ctx.register(buf, off)
        assert wc_multiset_gpu(buf, *ctx.wordcount(cap=1 << 17)) == want
        assert ctx.stats()["n_chunks"] >= 8
    with bk.Context(window_bytes=256 * 1024, n_slots=2, gather_mode=mode, test_delays=True) as ctx:
        ctx.register(gb, goff)
        assert np.array_equal(ctx.grep(b"bigk", cap=len(goff)), gwant)
    with bk.Context(window_bytes=512 * 1024, n_slots=2, gather_mode=mode, test_delays=True, record_size=16) as ctx:
        ctx.register(kv.view(np.uint8).reshape(-1), None, n_records=len(kv))
        out, cc, bc = ctx.partition(1024)
        assert np.array_equal(global_from_runs(out, cc), wout)
    # the drivers' setup on the compute stream (centroid upload, aggregate / table / cursor memsets)
    # is delayed ~2 ms behind the chunk streams: every chunk stage must still wait for it
    g = gen.groupby(n=100_000, stride=64)
    wc_, wq, wa = oracle.groupby(g, 100_000, 64, 4096)
    with bk.Context(window_bytes=512 * 1024, n_slots=2, gather_mode=mode, test_delays=True, record_size=64) as ctx:
        ctx.register(g, None, n_records=100_000)
        c, q, a = ctx.groupby(4096)
        assert np.array_equal(c, wc_) and np.array_equal(q, wq) and np.allclose(a, wa, rtol=1e-5, atol=0)
    x = gen.points(n=50_000)
    kc, _, kchk, kcid = oracle.kmeans(x, x[:64], want_cid=True)
    with bk.Context(window_bytes=512 * 1024, n_slots=2, gather_mode=mode, test_delays=True, record_size=64) as ctx:
        ctx.register(x.view(np.uint8).reshape(-1), None, n_records=50_000)
        cid = np.full(50_000, -1, np.int32)
        c, _, chk = ctx.kmeans(x[:64], cid=cid)
        assert np.array_equal(cid, kcid) and chk == kchk and np.array_equal(c, kc)
    d = gen.dna(n=4_000)
    okm, oct_ = oracle.kmer(d, 4_000, k=31)
    with bk.Context(window_bytes=256 * 1024, n_slots=2, gather_mode=mode, test_delays=True, record_size=256) as ctx:
        ctx.register(d, None, n_records=4_000)
        km, ct, _ = ctx.kmer(k=31, cap=1 << 20)
    o = np.argsort(km)
    assert np.array_equal(km[o], okm) and np.array_equal(ct[o], oct_)


@pytest.mark.parametrize("mode", ["fused", "zc"])
@pytest.mark.parametrize("where", ["kept_pinned_host", "device", "pageable_host"])
def test_wordcount_results_stored_by_the_compaction(mode, where):
    """k_wc_compact stores the distinct words straight into the caller's arrays when kernels can reach
    all of them (kept-pinned host memory through its mapped alias, device tensors); pageable host
    arrays get a copy after the run. Same multiset either way, replayed graphs included."""
    import torch
    buf, off = gen.text(cap_bytes=3 * MIB)
    want = oracle.wc(buf, off)
    cap = 1 << 18
    if where == "device":
        out = (torch.zeros(cap, dtype=torch.int64, device="cuda"), torch.zeros(cap, dtype=torch.int32, device="cuda"),
               torch.zeros(cap, dtype=torch.int64, device="cuda"), torch.zeros(cap, dtype=torch.int64, device="cuda"),
               torch.zeros(cap, dtype=torch.int64, device="cuda"))
    else:
        out = (np.zeros(cap, np.uint64), np.zeros(cap, np.uint32), np.zeros(cap, np.uint64))
    with bk.Context(window_bytes=2 * MIB, gather_mode=mode, keep_outputs_pinned=where == "kept_pinned_host") as ctx:
        ctx.register(buf, off)
        for _ in range(3):
            r = ctx.wordcount(out=out)
            o, ln, cnt = r[:3]
            if where == "device":
                o, ln, cnt = (o.cpu().numpy().view(np.uint64), ln.cpu().numpy().view(np.uint32),
                              cnt.cpu().numpy().view(np.uint64))
                h1, h2 = r[3].cpu().numpy(), r[4].cpu().numpy()
                assert len(h1) == len(o) and np.all(h1 != 0)
            assert wc_multiset_gpu(buf, o, ln, cnt) == want
            for a in out:
                a[:] = 0


def test_wordcount_direct_store_capacity_error_then_recovers():
    """Kept-pinned result arrays smaller than the vocabulary: BK_E_CAPACITY, then the same context
    with large enough arrays (another captured graph) is exact."""
    buf, off = gen.text(cap_bytes=1 * MIB)
    want = oracle.wc(buf, off)
    small = (np.zeros(100, np.uint64), np.zeros(100, np.uint32), np.zeros(100, np.uint64))
    big = (np.zeros(1 << 17, np.uint64), np.zeros(1 << 17, np.uint32), np.zeros(1 << 17, np.uint64))
    with bk.Context(window_bytes=2 * MIB, keep_outputs_pinned=True) as ctx:
        ctx.register(buf, off)
        with pytest.raises(bk.BkError) as e:
            ctx.wordcount(out=small)
        assert e.value.status == bk.BK_E_CAPACITY
        assert wc_multiset_gpu(buf, *ctx.wordcount(out=big)) == want


@pytest.mark.parametrize("env", [{"BK_FUSED_FEED": "dma", "BK_FUSED_BATCHES": "2"},
                                 {"BK_FUSED_FEED": "dma", "BK_FUSED_BATCHES": "5"},
                                 {"BK_FUSED_LOADERS": "1", "BK_FUSED_UNIT": "4096"},
                                 {"BK_FUSED_LOADERS": "9", "BK_FUSED_UNIT": "65536"}])
def test_wordcount_fused_knobs(monkeypatch, env):
    """The single launch's tuning knobs (copy-engine feed and its batch slots, loader count, unit
    size) change the schedule, never the table."""
    for k, v in env.items():
        monkeypatch.setenv(k, v)
    buf, off = gen.text(cap_bytes=3 * MIB)
    want = oracle.wc(buf, off)
    with bk.Context(window_bytes=2 * MIB, gather_mode="fused") as ctx:
        ctx.register(buf, off)
        for _ in range(2):
            assert wc_multiset_gpu(buf, *ctx.wordcount(cap=1 << 18)) == want


@pytest.mark.parametrize("cfg", ["1", "2", "3", "4", "5", "6", "7", "8"])
def test_host_packer_prefetch_configs(monkeypatch, cfg):
    """Every host-packer configuration (BK_PACK_CFG: prefetch distances; 7, 8 with 32-B AVX2 copies)
    packs the same bytes: grep keys of variable records (2 words per field), sparse group-by fields
    (1 word) and k-mer sequence fields (6 words) through CPU assembly."""
    monkeypatch.setenv("BK_PACK_CFG", cfg)
    gb, goff = gen.grep_records(max_bytes=4 * MIB)
    with bk.Context(window_bytes=1 * MIB, gather_mode="cpu") as ctx:
        ctx.register(gb, goff)
        assert np.array_equal(ctx.grep(b"bigk", cap=len(goff)), oracle.grep(gb, goff, b"bigk"))
    g = gen.groupby(n=60_000, stride=64)
    wc_, wq, wa = oracle.groupby(g, 60_000, 64, 4096)
    with bk.Context(window_bytes=1 * MIB, record_size=64, gather_mode="cpu") as ctx:
        ctx.register(g, None, n_records=60_000)
        c, q, a = ctx.groupby(4096)
        assert np.array_equal(c, wc_) and np.array_equal(q, wq) and np.allclose(a, wa, rtol=1e-5, atol=0)
    d = gen.dna(n=6_000)
    okm, oct_ = oracle.kmer(d, 6_000, k=31)
    with bk.Context(window_bytes=1 * MIB, record_size=256, gather_mode="cpu") as ctx:
        ctx.register(d, None, n_records=6_000)
        km, ct, _ = ctx.kmer(k=31, cap=1 << 20)
    o = np.argsort(km)
    assert np.array_equal(km[o], okm) and np.array_equal(ct[o], oct_)
