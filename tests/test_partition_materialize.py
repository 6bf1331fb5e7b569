"""bk_partition_materialize (host side, no GPU): chunk-major bucket-sorted runs -> the O4 order.

The runs are built here from the oracle itself (each chunk partitioned on its own, stable), which is
exactly what BK_K_PARTITION leaves in out_records (tests/test_gpu_parity.py checks that part on the
GPU); the materialised array must equal the oracle's partition of the whole data set."""
import numpy as np
import pytest

import gen
import oracle
from paper_conf_ipps_mokhtaris14_b200 import bk


def chunk_major(kv, B, bounds):
    outs, counts = [], []
    for lo, hi in zip(bounds[:-1], bounds[1:]):
        boff, part = oracle.partition(kv[lo:hi], B)
        outs.append(part)
        counts.append(np.diff(boff))
    return np.concatenate(outs), np.array(counts, np.uint64).reshape(len(outs), B)


@pytest.mark.parametrize("n,B,C", [(100_003, 1024, 7), (5000, 1, 3), (777, 4096, 5), (0, 64, 0), (64, 16, 64)])
def test_materialize_equals_oracle(n, B, C):
    kv = gen.kv(n=n) if n else np.zeros((0, 2), np.uint64)
    bounds = np.linspace(0, n, C + 1).astype(np.int64) if C else np.array([0])
    runs, cc = chunk_major(kv, B, bounds) if C else (kv, np.zeros((0, B), np.uint64))
    got = bk.partition_materialize(runs, cc, threads=4)
    boff, want = oracle.partition(kv, B)
    assert np.array_equal(got, want)


def test_materialize_two_ranks_into_one_array():
    """Multi-GPU layout: each rank passes its global bucket offsets (merge_partition_offsets) and
    fills a disjoint share of one array; the union is the global stable partition."""
    n, B = 60_001, 256
    kv = gen.kv(n=n)
    mid = n // 2
    shards = [(0, mid), (mid, n)]
    per = []
    for lo, hi in shards:
        runs, cc = chunk_major(kv[lo:hi], B, np.linspace(0, hi - lo, 5).astype(np.int64))
        per.append((runs, cc, cc.sum(0).astype(np.int64)))
    tot = per[0][2] + per[1][2]
    boff = np.concatenate([[0], np.cumsum(tot)])
    dst = np.zeros((n, 2), np.uint64)
    below = np.zeros(B, np.int64)
    for runs, cc, bc in per:
        bk.partition_materialize(runs, cc, bucket_start=(boff[:-1] + below).astype(np.uint64), dst=dst, threads=3)
        below += bc
    assert np.array_equal(dst, oracle.partition(kv, B)[1])


def test_materialize_errors():
    with pytest.raises(bk.BkError) as e:
        bk.partition_materialize(np.zeros((1, 2), np.uint64), np.zeros((1, 0), np.uint64))
    assert e.value.status == bk.BK_E_INVAL
