"""Pins for the layout oracle O-L (address generation + assembly; PAPER.md:381-392, P:426-430,
P:546-555; SURVEY O-L, A3, A4) and the pattern detector O-P."""
import numpy as np
import pytest

import gen
import oracle
from _pins import golden


def accessed(buf: bytes, off, n, nbytes, rec_size, extents, lo, hi) -> bytes:
    out = b""
    for r in range(lo, hi):
        s = int(off[r]) if off is not None else r * rec_size
        e = (int(off[r + 1]) if r + 1 < n else nbytes) if off is not None else s + rec_size
        if not extents:
            out += buf[s:e]
        else:
            for eo, el in extents:
                out += buf[s + eo: s + eo + el]
    return out


def deinterleave(stage: np.ndarray, lane_bytes, L):
    """Read lane t's bytes back out of the warp tiles: independent of how they were written."""
    st = stage.tobytes()
    lanes, base = [], 0
    for w in range(L // 32):
        K = max((int(b) + 15) // 16 for b in lane_bytes[32 * w: 32 * w + 32])
        tile = np.frombuffer(st[base: base + 512 * K], np.uint8).reshape(K, 32, 16)
        for t in range(32):
            nb = int(lane_bytes[32 * w + t])
            lanes.append(tile[:, t, :].reshape(-1).tobytes()[:nb])
            assert not tile[:, t, :].reshape(-1)[nb:].any(), "holes must be zero"
        base += 512 * K
    assert base == len(st)
    return lanes


CASES = [
    ("wc", None, 0),
    ("grep", [(16, 32)], 0),
    ("groupby_sparse", [(0, 16)], 64),
    ("dup_extents", [(8, 4), (0, 12), (8, 4)], 16),   # duplicates repeat
]


def dataset(kind):
    if kind == "wc":
        buf, off = gen.text(cap_bytes=60000)
        return buf, off, len(off), len(buf), 0
    if kind == "grep":
        buf, off = gen.grep_records(n=700)
        return buf, off, len(off), len(buf), 0
    if kind == "groupby_sparse":
        buf = gen.groupby(n=900, stride=64)
        return buf, None, 900, len(buf), 64
    buf = gen.groupby(n=777, stride=16)
    return buf, None, 777, len(buf), 16


@pytest.mark.parametrize("kind,extents,_", CASES)
@pytest.mark.parametrize("L", [32, 96])
def test_layout_roundtrip_and_balance(kind, extents, _, L):
    buf, off, n, nbytes, rs = dataset(kind)
    budget = 8192
    bounds = oracle.plan_chunks(off, n, nbytes, rs, extents, budget)
    b = buf.tobytes()
    for c in range(len(bounds) - 1):
        lo, hi = int(bounds[c]), int(bounds[c + 1])
        stage, lf, ln, lb = oracle.layout(buf, off, n, nbytes, rs, extents, lo, hi, L)
        # lanes are contiguous, ordered, and cover [lo, hi)
        assert lf[0] == lo and int(lf[-1] + ln[-1]) == hi
        assert np.all(lf[1:] == lf[:-1] + ln[:-1])
        # de-interleaving the tiles returns exactly the accessed bytes in record order (I3, I5)
        lanes = deinterleave(stage, lb, L)
        assert b"".join(lanes) == accessed(b, off, n, nbytes, rs, extents, lo, hi)
        for t in range(L):
            assert lanes[t] == accessed(b, off, n, nbytes, rs, extents, int(lf[t]), int(lf[t] + ln[t]))
        # balance: no lane holds more than its share plus one record
        total = sum(int(v) for v in lb)
        maxrec = max((len(accessed(b, off, n, nbytes, rs, extents, r, r + 1)) for r in range(lo, hi)), default=0)
        assert max(int(v) for v in lb) <= -(-total // L) + maxrec


def test_layout_special_case_is_a_transpose():
    """One 16k-byte record per lane: the layout is the paper's buf[counter][tid] transpose
     with 16-byte elements, i.e. a plain numpy transpose per warp tile."""
    k, L = 3, 64
    buf = np.arange(L * 16 * k, dtype=np.uint32).astype(np.uint8)
    stage, lf, ln, lb = oracle.layout(buf, None, L, len(buf), 16 * k, None, 0, L, L)
    words = buf.reshape(L // 32, 32, k, 16)          # [warp][lane][counter][byte]
    assert stage.tobytes() == words.transpose(0, 2, 1, 3).tobytes()   # [warp][counter][lane][byte]
    assert list(ln) == [1] * L


def test_chunk_plan_is_greedy_whole_records():
    buf, off = gen.text(cap_bytes=50000)
    n, nb = len(off), len(buf)
    ends = np.append(off[1:], nb).astype(np.int64)
    lens = ends - off.astype(np.int64)
    for budget in [int(lens.max()), 1000, 4096, 1 << 20]:
        bounds = oracle.plan_chunks(off, n, nb, 0, None, budget)
        assert bounds[0] == 0 and bounds[-1] == n
        for c in range(len(bounds) - 1):
            lo, hi = int(bounds[c]), int(bounds[c + 1])
            assert hi > lo and lens[lo:hi].sum() <= budget
            if hi < n:
                assert lens[lo:hi + 1].sum() > budget  # maximal
    with pytest.raises(OverflowError):
        oracle.plan_chunks(off, n, nb, 0, None, int(lens.max()) - 1)  # BK_E_RANGE (A18)
    assert list(oracle.plan_chunks(np.zeros(0, np.uint64), 0, 0, 0, None, 100)) == [0]


def test_empty_records_and_empty_chunk_lanes():
    off = np.array([0, 0, 0, 5, 5], np.uint64)
    buf = np.frombuffer(b"hello", np.uint8)
    stage, lf, ln, lb = oracle.layout(buf, off, 5, 5, 0, None, 0, 5, 32)
    assert int(ln.sum()) == 5 and int(lb.sum()) == 5
    assert stage.tobytes()[:16] == b"hello" + b"\x00" * 11 or b"hello" in stage.tobytes()


def test_pattern_paper_example():
    g = golden("pattern_example.json")
    for key in ("decimal_reading", "hex_reading"):
        base, strides = oracle.pattern(g[key]["addrs"])
        assert base == g[key]["base"] and strides == g[key]["strides"]


def test_pattern_online_detect_then_verify():
    g = golden("pattern_example.json")
    # the paper's example, extended: the detected stride holds for every later address
    a = list(range(100, 100 + 5 * 40, 5))
    assert oracle.pattern_online(a, T=4) == (100, [5])
    assert oracle.pattern_online(g["decimal_reading"]["addrs"], T=8) == (100, [5])
    # a late mismatch abandons the pattern ("If it does not, then address generation
    # is started again, this time without attempting to identify a pattern")
    assert oracle.pattern_online(a[:30] + [a[29] + 7] + a[31:], T=4) is None
    # detection sees only the first T: a longer true period is missed (fallback), unlike the
    # whole-list detector
    b = [0, 1, 2, 3, 10, 11, 12, 13, 20, 21, 22, 23]
    assert oracle.pattern(b) == (0, [1, 1, 1, 7])
    assert oracle.pattern_online(b, T=4) is None
    assert oracle.pattern_online(b, T=8) == (0, [1, 1, 1, 7])
    # byte addresses of a contiguous text lane (WC, 1-byte elements) and fp32 fields of 64-B
    # records (K-means, 4-byte elements) reduce to one stride
    assert oracle.pattern_online(list(range(1000, 1300)), T=8) == (1000, [1])
    assert oracle.pattern_online([r * 64 + 4 * j for r in range(10) for j in range(16)], T=8) == (0, [4])
    # sparse group-by: {key, qty, amount} = 4 + 4 + 8 bytes at +0 of 64-B records, 4-byte elements
    assert oracle.pattern_online([r * 64 + e for r in range(20) for e in (0, 4, 8, 12)], T=8) == (0, [4, 4, 4, 52])
    assert oracle.pattern_online([7], T=8) is None and oracle.pattern_online([], T=8) is None


def test_pattern_fallback_and_multi_stride():
    assert oracle.pattern([10, 13, 20, 27, 40]) is None  # no period <= 4 fits -> explicit list
    assert oracle.pattern([0, 4, 8, 64, 68, 72, 128], pmax=4) == (0, [4, 4, 56])
    assert oracle.pattern([5]) is None
    # K-means x/y/z of 32-byte particles: strides 4, 4, 24
    a = [i * 32 + f for i in range(6) for f in (0, 4, 8)]
    assert oracle.pattern(a) == (0, [4, 4, 24])
