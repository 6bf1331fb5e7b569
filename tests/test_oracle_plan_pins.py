"""Independent pins of the two planning rules the oracle fixes (readings A3, A4) and the
GPU was written to match (VERDICT r1 "weak" 1):

  A3 chunk plan (Fig. 3's `counter < addrBufSize` read as whole records only):
     a chunk is the LONGEST run of whole records, starting where the previous one ended, whose
     accessed bytes fit the budget (greedy, maximal); a record larger than the budget is BK_E_RANGE.
  A4 lane rule (each thread a contiguous record range, balanced by accessed bytes):
     first(t) = min{ r : A(lo, r) >= floor(t * A(lo, hi) / L) },  first(L) = hi.

Each is restated here in a different way than oracle.c computes it (numpy prefix sums + bisect,
a running greedy in Python, hand-computed tables), so an off-by-one in either (ceil vs floor,
< vs <=, the record that overflows) fails one of these tests."""
import bisect

import numpy as np
import pytest

import gen
import oracle


def accessed_per_record(off, n, nbytes, rec_size, extents):
    if off is not None:
        ends = np.append(off[1:].astype(np.int64), nbytes)
        lens = ends - off.astype(np.int64)
    else:
        lens = np.full(n, rec_size, np.int64)
    if not extents:
        return lens
    assert all(eo + el <= l for l in lens for eo, el in extents)
    return np.full(n, sum(el for _, el in extents), np.int64)


def greedy_bounds(acc, budget):
    """A3 restated: walk the records once, closing a chunk when the next record would not fit."""
    bounds, used = [0], 0
    for r, a in enumerate(acc):
        if a > budget:
            return None
        if used + a > budget:
            bounds.append(r)
            used = 0
        used += a
    if bounds[-1] != len(acc):
        bounds.append(len(acc))
    return bounds


PLAN_CASES = [
    ("grep_key", [(16, 32)]),          # variable records, one extent
    ("grep_multi", [(16, 8), (40, 8)]),
    ("text_whole", None),              # variable records, whole
    ("sparse64", [(0, 16)]),           # fixed records, one extent
    ("dup16", [(8, 4), (0, 12), (8, 4)]),
    ("kmer", [(16, 96)]),
]


def plan_data(kind):
    if kind in ("grep_key", "grep_multi"):
        buf, off = gen.grep_records(n=3000)
        return off, len(off), len(buf), 0
    if kind == "text_whole":
        buf, off = gen.text(cap_bytes=80_000)
        return off, len(off), len(buf), 0
    if kind == "sparse64":
        return None, 2500, 2500 * 64, 64
    if kind == "kmer":
        return None, 1000, 1000 * 256, 256
    return None, 4001, 4001 * 16, 16


@pytest.mark.parametrize("kind,extents", PLAN_CASES)
@pytest.mark.parametrize("budget", [96, 100, 1000, 4096, 12_345])
def test_plan_chunks_with_extents_is_the_greedy_maximal_plan(kind, extents, budget):
    off, n, nbytes, rs = plan_data(kind)
    acc = accessed_per_record(off, n, nbytes, rs, extents)
    want = greedy_bounds(acc, budget)
    if want is None:
        with pytest.raises(OverflowError):
            oracle.plan_chunks(off, n, nbytes, rs, extents, budget)
        return
    got = [int(x) for x in oracle.plan_chunks(off, n, nbytes, rs, extents, budget)]
    assert got == want
    # maximality stated directly: every chunk fits, and one more record would not
    pre = np.concatenate([[0], np.cumsum(acc)])
    for lo, hi in zip(got[:-1], got[1:]):
        assert hi > lo and pre[hi] - pre[lo] <= budget
        if hi < n:
            assert pre[hi + 1] - pre[lo] > budget


def test_plan_chunks_hand_table():
    """Fixed 16-B records, extent of 12 B (E = 12), budget 40: chunks of 3 records (36 <= 40 < 48)."""
    got = [int(x) for x in oracle.plan_chunks(None, 10, 160, 16, [(2, 12)], 40)]
    assert got == [0, 3, 6, 9, 10]
    # budget exactly 3 records' worth: still 3 per chunk (<=, not <)
    assert [int(x) for x in oracle.plan_chunks(None, 10, 160, 16, [(2, 12)], 36)] == [0, 3, 6, 9, 10]
    # one byte less: 2 per chunk
    assert [int(x) for x in oracle.plan_chunks(None, 10, 160, 16, [(2, 12)], 35)] == [0, 2, 4, 6, 8, 10]
    with pytest.raises(OverflowError):
        oracle.plan_chunks(None, 10, 160, 16, [(2, 12)], 11)


def lanes_by_bisect(acc_chunk, lo, L):
    """A4 restated: the prefix sums of the chunk are sorted, so first(t) is a bisect_left of the
    target floor(t*A/L) into them (Python ints: no overflow, exact floor)."""
    pre = [0]
    for a in acc_chunk:
        pre.append(pre[-1] + int(a))
    A = pre[-1]
    first = [lo + bisect.bisect_left(pre, (t * A) // L) for t in range(L)] + [lo + len(acc_chunk)]
    return first


@pytest.mark.parametrize("kind,extents", PLAN_CASES)
@pytest.mark.parametrize("L", [32, 64, 288])
def test_layout_lane_rule_is_bisect_of_floor_target(kind, extents, L):
    off, n, nbytes, rs = plan_data(kind)
    acc = accessed_per_record(off, n, nbytes, rs, extents)
    bounds = oracle.plan_chunks(off, n, nbytes, rs, extents, 6000)
    buf = np.zeros(nbytes, np.uint8)
    for lo, hi in zip(bounds[:-1].astype(int), bounds[1:].astype(int)):
        _, lf, ln, lb = oracle.layout(buf, off, n, nbytes, rs, extents, lo, hi, L, with_stage=False)
        first = lanes_by_bisect(acc[lo:hi], lo, L)
        assert [int(x) for x in lf] == first[:L]
        assert [int(x) for x in ln] == [first[t + 1] - first[t] for t in range(L)]
        assert [int(x) for x in lb] == [int(acc[first[t]: first[t + 1]].sum()) for t in range(L)]


def test_layout_lane_rule_hand_table():
    """Ten 1-byte records over L = 32 lanes: target(t) = floor(10 t / 32), so lane t starts at record
    floor(10 t / 32) — lanes 0-3 start at 0 (only lane 3 owns it: lanes 0-2 are empty), lane 4 at 1 (40/32 = 1.25), ...
    A ceil rule would start lane 4 at record 2; a '>' instead of '>=' would shift every lane."""
    buf = np.frombuffer(b"abcdefghij", np.uint8)
    _, lf, ln, lb = oracle.layout(buf, None, 10, 10, 1, None, 0, 10, 32, with_stage=False)
    want_first = [(10 * t) // 32 for t in range(32)]
    assert [int(x) for x in lf] == want_first
    want_n = [(want_first[t + 1] if t + 1 < 32 else 10) - want_first[t] for t in range(32)]
    assert [int(x) for x in ln] == want_n
    # spelled out: records 0..9 are owned by lanes 3, 6, 9, 12, 15, 19, 22, 25, 28, 31 (the last t with floor(10t/32) <= r)
    owners = [t for t in range(32) for _ in range(want_n[t])]
    assert owners == [3, 6, 9, 12, 15, 19, 22, 25, 28, 31]
    assert sum(want_n) == 10 and list(lb) == want_n


def test_layout_lane_rule_exact_split():
    """m = k * L equal records: every lane owns exactly k consecutive records (target t*k*s)."""
    k, L, s = 3, 64, 24
    buf = np.zeros(k * L * s, np.uint8)
    _, lf, ln, lb = oracle.layout(buf, None, k * L, len(buf), s, None, 0, k * L, L, with_stage=False)
    assert list(lf) == [k * t for t in range(L)] and set(ln) == {k} and set(lb) == {k * s}


def test_layout_lane_rule_empty_records_go_to_the_earliest_lane():
    """Zero-length records sit at a prefix equal to the target of the lanes before them: with
    bisect_left they belong to the earliest lane whose target they reach."""
    off = np.array([0, 0, 0, 5, 5, 9], np.uint64)   # lengths 0, 0, 5, 0, 4, 3 (nbytes 12)
    buf = np.frombuffer(b"hello" + b"worl" + b"d!!", np.uint8)
    acc = [0, 0, 5, 0, 4, 3]
    _, lf, ln, lb = oracle.layout(buf, off, 6, 12, 0, None, 0, 6, 32, with_stage=False)
    assert [int(x) for x in lf] == lanes_by_bisect(acc, 0, 32)[:32]
    assert lf[0] == 0 and int(ln.sum()) == 6 and int(lb.sum()) == 12
