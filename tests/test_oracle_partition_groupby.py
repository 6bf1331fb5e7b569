"""Pins for oracle O4 (hash partition, A14) and O5 (group-by sum, A15)."""
import struct
from collections import defaultdict

import numpy as np
import pytest

import gen
import oracle
from _pins import mix64


def bucket(key: int, B: int) -> int:
    bits = B.bit_length() - 1
    return mix64(key) >> (64 - bits) if bits else 0


@pytest.mark.parametrize("B", [1, 2, 1024])
def test_partition_brute_force(B):
    kv = gen.kv(n=3000)
    boff, out = oracle.partition(kv, B)
    # brute force: for b in 0..B-1 scan all records in input order
    exp = [tuple(r) for b in range(B) for r in kv.tolist() if bucket(r[0], B) == b]
    assert [tuple(r) for r in out.tolist()] == exp
    assert boff[0] == 0 and boff[-1] == len(kv)
    for b in range(0, B, max(1, B // 16)):
        seg = out[int(boff[b]): int(boff[b + 1])]
        assert all(bucket(int(k), B) == b for k in seg[:, 0])
        assert np.all(np.diff(seg[:, 1].astype(np.int64)) > 0)  # stable: value = original index


def test_partition_invariants_and_identity():
    kv = gen.kv(n=50000)
    boff, out = oracle.partition(kv, 1024)
    assert np.array_equal(np.sort(out[:, 1]), np.arange(50000, dtype=np.uint64))
    assert np.array_equal(np.sort(out[:, 0]), np.sort(kv[:, 0]))
    assert np.all(np.diff(boff.astype(np.int64)) >= 0)
    boff1, out1 = oracle.partition(kv, 1)
    assert np.array_equal(out1, kv) and list(boff1) == [0, 50000]
    with pytest.raises(ValueError):
        oracle.partition(kv, 1000)
    # duplicate keys all land in one bucket, in input order
    dup = np.array([[7, i] for i in range(10)], np.uint64)
    b2, o2 = oracle.partition(dup, 1024)
    assert np.array_equal(o2, dup)


def recs(rows, stride=16):
    out = bytearray()
    for k, q, a in rows:
        out += struct.pack("<IId", k, q, a) + b"\xab" * (stride - 16)
    return np.frombuffer(bytes(out), np.uint8)


@pytest.mark.parametrize("stride", [16, 64])
def test_groupby_brute_force(stride):
    n = 4000
    buf = gen.groupby(n=n, G=64, stride=stride)
    count, qty, amt = oracle.groupby(buf, n, stride, 64)
    c, q, a = defaultdict(int), defaultdict(int), defaultdict(float)
    cents = defaultdict(int)
    for i in range(n):
        k, qq, aa = struct.unpack_from("<IId", buf, i * stride)
        c[k] += 1; q[k] += qq; a[k] += aa
        cents[k] += round(aa * 100)
    for k in range(64):
        assert count[k] == c[k] and qty[k] == q[k] and amt[k] == a[k]
        assert abs(amt[k] - cents[k] / 100) <= 1e-9 * max(1.0, cents[k] / 100)
    assert count.sum() == n


def test_groupby_special_cases():
    one = recs([(0, 5, 1.25), (0, 7, 2.5), (0, 1, 0.0)])
    count, qty, amt = oracle.groupby(one, 3, 16, 1)
    assert list(count) == [3] and list(qty) == [13] and list(amt) == [3.75]
    last = recs([(4095, 1, 0.5)])
    count, _, _ = oracle.groupby(last, 1, 16, 4096)
    assert count[4095] == 1 and count.sum() == 1
    with pytest.raises(ValueError):
        oracle.groupby(recs([(4096, 1, 0.5)]), 1, 16, 4096)
    count, qty, amt = oracle.groupby(np.zeros(0, np.uint8), 0, 16, 8)
    assert not count.any() and not amt.any()


def test_groupby_sort_then_sum_equivalence():
    n = 20000
    buf = gen.groupby(n=n, G=4096, zipf=True)
    count, qty, amt = oracle.groupby(buf, n, 16, 4096)
    a = np.frombuffer(buf.tobytes(), dtype=np.dtype([("k", "<u4"), ("q", "<u4"), ("a", "<f8")]))
    order = np.argsort(a["k"], kind="stable")
    ks = a["k"][order]
    bounds = np.searchsorted(ks, np.arange(4097))
    for k in range(0, 4096, 37):
        seg = order[bounds[k]: bounds[k + 1]]
        assert count[k] == len(seg) and qty[k] == int(a["q"][seg].astype(np.uint64).sum())
        np.testing.assert_allclose(amt[k], a["a"][seg].sum(), rtol=1e-12)
    assert count[0] > count[4095]  # Zipf skew
