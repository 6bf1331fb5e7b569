"""GPU parity of f4 (k-mer counting over DNA read records) against oracle O6."""
import numpy as np
import pytest

import gen
import oracle
from paper_conf_ipps_mokhtaris14_b200 import bk

pytestmark = pytest.mark.gpu
MIB = 1 << 20


def sorted_pairs(km, ct):
    o = np.argsort(km)
    return km[o], ct[o]


@pytest.mark.parametrize("k,mode", [(31, "hybrid"), (21, "zc"), (13, "dense"), (31, "cpu"), (1, "zc")])
def test_kmer_matches_oracle(k, mode):
    n = 40_000
    buf = gen.dna(n=n, genome_len=1 << 18, err_pm=2, n_pm=3)
    wk, wc = oracle.kmer(buf, n, k)
    with bk.Context(window_bytes=2 * MIB, gather_mode=mode, record_size=256) as ctx:
        ctx.register(buf, None, n_records=n)
        km, ct, total = ctx.kmer(k=k, table_slots=1 << 22)
        st = ctx.stats()
    assert st["n_chunks"] >= 4
    gk, gc = sorted_pairs(km, ct)
    assert np.array_equal(gk, wk) and np.array_equal(gc, wc)
    assert total == int(wc.sum())
    if mode == "zc":
        assert st["bytes_accessed"] == 96 * n   # 37.5% of the 256-B records (Table I DNA: 36%)


def test_kmer_errors():
    buf = gen.dna(n=1000)
    with bk.Context(window_bytes=1 * MIB, record_size=256) as ctx:
        ctx.register(buf, None, n_records=1000)
        for kw in ({"k": 0}, {"k": 32}, {"seq_len": 90}, {"seq_off": 200}, {"table_slots": 1000}):
            with pytest.raises(bk.BkError):
                ctx.kmer(**kw)
        with pytest.raises(bk.BkError) as e:
            ctx.kmer(k=31, table_slots=1 << 10)
        assert e.value.status == bk.BK_E_CAPACITY


def _windows(seq: np.ndarray, k: int):
    """All k-windows of a block of reads (uint8 [reads, L]): packed values (A=0 C=1 G=2 T=3, first
    base most significant) and validity (every base in ACGT). Plain definition, no rolling."""
    code = np.full(seq.shape, 255, np.uint8)
    for i, ch in enumerate(b"ACGT"):
        code[seq == ch] = i
    ok = code != 255
    W = seq.shape[1] - k + 1
    val = np.zeros((seq.shape[0], W), np.uint64)
    valid = np.ones((seq.shape[0], W), bool)
    for i in range(k):
        val <<= np.uint64(2)
        val |= code[:, i:i + W] & np.uint8(3)
        valid &= ok[:, i:i + W]
    return val, valid


def test_kmer_bench_scale_sampled():
    """The bench configuration (4 GiB of reads, 2 GiB window, k = 31, AUTO gather): the total
    equals the number of valid windows counted from the definition, the counts sum to it, and
    64 sampled k-mers have exactly the counts a brute-force recount over every read gives."""
    k, n = 31, (4 << 30) // 256
    buf = gen.dna(gen.SEED_DNA, first=0, n=n, genome_len=1 << 25, err_pm=1, n_pm=2, threads=16)
    with bk.Context(window_bytes=2 << 30, record_size=256) as ctx:
        ctx.register(buf, None, n_records=n)
        km, ct, total = ctx.kmer(k=k, table_slots=1 << 28, cap=1 << 27)
    assert int(ct.sum()) == total
    rng = np.random.default_rng(7)
    pick = rng.choice(len(km), 64, replace=False)
    want = {int(km[i]): int(ct[i]) for i in pick}
    keys = np.array(sorted(want), np.uint64)
    seqs = buf.reshape(n, 256)[:, 16:112]

    def block(lo):  # numpy releases the GIL: blocks recount in parallel
        val, valid = _windows(seqs[lo:lo + (1 << 18)], k)
        v = val[valid]
        idx = np.searchsorted(keys, v)
        idx[idx == len(keys)] = 0
        m = keys[idx] == v
        return int(valid.sum()), np.bincount(idx[m], minlength=len(keys))

    from concurrent.futures import ThreadPoolExecutor
    with ThreadPoolExecutor(8) as ex:
        parts = list(ex.map(block, range(0, n, 1 << 18)))
    n_valid = sum(p[0] for p in parts)
    hits = sum(p[1] for p in parts)
    assert total == n_valid
    assert {int(key): int(h) for key, h in zip(keys, hits)} == want


@pytest.mark.parametrize("n,slots", [(60, 1 << 13), (6000, 1 << 18), (6000, 1 << 22)])
def test_kmer_skewed_buckets_and_region_sizes(n, slots):
    """Two-phase counting under skew: half the reads are poly-A (one k-mer for every window: its
    region's bucket overflows and the rest goes to the region directly), the rest random; a table of
    one region (2^13 slots), a few regions, and many."""
    buf = gen.dna(n=n, genome_len=1 << 16, err_pm=2, n_pm=3).reshape(n, 256).copy()
    buf[::2, 16:112] = ord("A")
    buf = buf.reshape(-1)
    wk, wc = oracle.kmer(buf, n, 31)
    assert len(wk) * 2 < slots
    with bk.Context(window_bytes=1 * MIB, record_size=256, gather_mode="zc") as ctx:
        ctx.register(buf, None, n_records=n)
        km, ct, total = ctx.kmer(k=31, table_slots=slots, cap=1 << 20)
    gk, gc = sorted_pairs(km, ct)
    assert np.array_equal(gk, wk) and np.array_equal(gc, wc) and total == int(wc.sum())


@pytest.mark.parametrize("flush_every,split_each", [(1, "0"), (3, "0"), (1, "1"), (2, "1")])
def test_kmer_mid_run_flushes(monkeypatch, flush_every, split_each):
    """Mid-run flushes (every F chunks: the regions are written back with their 64-bit counts and
    reloaded by the next flush) and the per-chunk coarse -> fine split give the oracle's table."""
    monkeypatch.setenv("BK_KMER_F", str(flush_every))
    monkeypatch.setenv("BK_KMER_SPLIT_EACH", split_each)
    n = 30_000
    buf = gen.dna(n=n, genome_len=1 << 16, err_pm=2, n_pm=3)
    wk, wc = oracle.kmer(buf, n, 31)
    with bk.Context(window_bytes=2 * MIB, record_size=256, gather_mode="hybrid") as ctx:
        ctx.register(buf, None, n_records=n)
        for _ in range(2):   # the second run replays the captured graph
            km, ct, total = ctx.kmer(k=31, table_slots=1 << 22)
            gk, gc = sorted_pairs(km, ct)
            assert np.array_equal(gk, wk) and np.array_equal(gc, wc) and total == int(wc.sum())
        assert ctx.stats()["n_chunks"] >= 4


@pytest.mark.parametrize("where", ["pinned_host", "device"])
def test_kmer_results_stored_by_the_flush(where):
    """The final flush stores the distinct k-mers straight into the caller's arrays when kernels can
    reach them: host arrays the context keeps pinned (mapped stores over PCIe) or device tensors."""
    import torch
    n = 20_000
    buf = gen.dna(n=n, genome_len=1 << 16, err_pm=2, n_pm=3)
    wk, wc = oracle.kmer(buf, n, 31)
    cap = 1 << 20
    if where == "device":
        out = (torch.zeros(cap, dtype=torch.int64, device="cuda"), torch.zeros(cap, dtype=torch.int64, device="cuda"))
    else:
        out = (np.zeros(cap, np.uint64), np.zeros(cap, np.uint64))
    with bk.Context(window_bytes=2 * MIB, record_size=256, keep_outputs_pinned=True) as ctx:
        ctx.register(buf, None, n_records=n)
        for _ in range(2):
            km, ct, total = ctx.kmer(k=31, table_slots=1 << 22, out=out)
            if where == "device":
                km, ct = km.cpu().numpy().view(np.uint64), ct.cpu().numpy().view(np.uint64)
            gk, gc = sorted_pairs(km, ct)
            assert np.array_equal(gk, wk) and np.array_equal(gc, wc) and total == int(wc.sum())
            out[0][:] = 0
            out[1][:] = 0


def test_kmer_direct_store_capacity_error_then_recovers():
    """Kept-pinned result arrays smaller than the distinct k-mers: BK_E_CAPACITY (the flush stored only
    what fits), then a run into large enough arrays on the same context is exact."""
    n = 5000
    buf = gen.dna(n=n, genome_len=1 << 16, err_pm=2, n_pm=3)
    wk, wc = oracle.kmer(buf, n, 31)
    small = (np.zeros(len(wk) // 2, np.uint64), np.zeros(len(wk) // 2, np.uint64))
    big = (np.zeros(len(wk) + 10, np.uint64), np.zeros(len(wk) + 10, np.uint64))
    with bk.Context(window_bytes=1 * MIB, record_size=256, keep_outputs_pinned=True) as ctx:
        ctx.register(buf, None, n_records=n)
        with pytest.raises(bk.BkError) as e:
            ctx.kmer(k=31, table_slots=1 << 20, out=small)
        assert e.value.status == bk.BK_E_CAPACITY
        km, ct, total = ctx.kmer(k=31, table_slots=1 << 20, out=big)
        gk, gc = sorted_pairs(km, ct)
        assert np.array_equal(gk, wk) and np.array_equal(gc, wc) and total == int(wc.sum())
