"""N>1 path on CPU: world_size-2 gloo processes run the sharding + merge logic of merge.py on
oracle-computed per-shard results and must reproduce the single-process answer exactly
(invariant I1: results independent of the GPU count P)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import gen
import oracle
from paper_conf_ipps_mokhtaris14_b200 import merge


def free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def word_key(w: bytes) -> int:
    import hashlib
    return int.from_bytes(hashlib.blake2b(w, digest_size=8).digest(), "little") >> 1


def worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        res = {}
        # group-by: shard, per-shard oracle, merge_sum
        n = 50_001
        lo, hi = merge.shard_range(n, rank, world)
        buf = gen.groupby(first=lo, n=hi - lo, G=256)
        c, q_, a = oracle.groupby(buf, hi - lo, 16, 256)
        t = torch.from_numpy(np.stack([c.astype(np.float64), q_.astype(np.float64), a]))
        res["groupby"] = merge.merge_sum(t).numpy()
        # k-means: counts/sums + checksum over shards with global first index
        n2 = 20_003
        lo2, hi2 = merge.shard_range(n2, rank, world)
        x = gen.points(first=lo2, n=hi2 - lo2)
        mu = gen.points(first=0, n=16)
        kc, ks, kchk, _ = oracle.kmeans(x, mu, first=lo2)
        res["kmeans"] = merge.merge_sum(torch.from_numpy(np.concatenate([kc.astype(np.float64), ks.ravel()]))).numpy()
        res["kmeans_chk"] = merge.merge_checksum(kchk)
        # grep: rank ranges of variable-length records, global offsets of the ascending lists
        first = 0
        for r in range(rank):
            first += gen.grep_count_for_bytes(gen.SEED_GREP, first, 300_000)
        gb, goff = gen.grep_records(first=first, max_bytes=300_000)
        idx = oracle.grep(gb, goff, b"bigk", first=first)
        off_, total = merge.merge_grep_offsets(len(idx))
        res["grep"] = (off_, total, idx)
        # partition: per-rank stable partition + global placement of runs
        n3 = 30_000
        lo3, hi3 = merge.shard_range(n3, rank, world)
        kv = gen.kv(first=lo3, n=hi3 - lo3)
        boff, out = oracle.partition(kv, 64)
        start, gboff = merge.merge_partition_offsets(np.diff(boff))
        res["partition"] = (start, gboff, boff, out)
        # word count: the all-gather of compacted per-rank rows (merge.gather_rows; the GPU merge by
        # key, bk_merge_counts, is covered by tests/test_gpu_merge.py): rows {key, len, count, rank, off}
        tb, toff = gen.text(gen.SEED_WC + rank, cap_bytes=20_000)
        raw = tb.tobytes()
        rows = [[word_key(w), len(w), c, rank, raw.find(w)] for w, c in oracle.wc(tb, toff)]
        t = torch.tensor(rows, dtype=torch.int64)
        g, counts, stride = merge.gather_rows(t, len(rows) - 3)   # a rank may send fewer rows than it holds
        res["wc"] = (g.numpy(), counts, stride, len(rows))
        q.put((rank, res))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_merge_matches_single_process(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = free_port()
    procs = [ctx.Process(target=worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    results = dict(q.get(timeout=240) for _ in procs)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    # group-by
    buf = gen.groupby(n=50_001, G=256)
    c, q_, a = oracle.groupby(buf, 50_001, 16, 256)
    for r in range(world):
        g = results[r]["groupby"]
        assert np.array_equal(g[0], c.astype(np.float64)) and np.array_equal(g[1], q_.astype(np.float64))
        np.testing.assert_allclose(g[2], a, rtol=1e-12)
    # k-means
    x = gen.points(n=20_003)
    kc, ks, kchk, _ = oracle.kmeans(x, gen.points(n=16))
    km = results[0]["kmeans"]
    assert np.array_equal(km[:16], kc.astype(np.float64))
    np.testing.assert_allclose(km[16:].reshape(16, 16), ks, rtol=1e-12)
    assert results[0]["kmeans_chk"] == results[1]["kmeans_chk"] == kchk
    # grep: concatenating rank lists at their offsets = the single-process answer
    total = results[0]["grep"][1]
    glob = np.empty(total, np.uint64)
    for r in range(world):
        off_, tot, idx = results[r]["grep"]
        glob[off_: off_ + len(idx)] = idx
    n_all = sum(len(results[r]["grep"][2]) for r in range(world))
    assert n_all == total
    first = 0
    segs = []
    for r in range(world):
        gb, goff = gen.grep_records(first=first, max_bytes=300_000)
        segs.append(oracle.grep(gb, goff, b"bigk", first=first))
        first += len(goff)
    assert np.array_equal(glob, np.concatenate(segs))
    # partition: placing each rank's bucket runs at start[b] rebuilds the global stable partition
    kv_all = gen.kv(n=30_000)
    wboff, wout = oracle.partition(kv_all, 64)
    glob = np.empty_like(wout)
    for r in range(world):
        start, gboff, boff, out = results[r]["partition"]
        assert np.array_equal(gboff, wboff)
        for b in range(64):
            seg = out[int(boff[b]): int(boff[b + 1])]
            glob[int(start[b]): int(start[b]) + len(seg)] = seg
    assert np.array_equal(glob, wout)
    # word count: the gathered segments hold every rank's first n rows, padded to the longest
    g, counts, stride, nrows = results[0]["wc"]
    assert np.array_equal(g, results[1]["wc"][0]) and stride == max(counts)
    merged = {}
    for r in range(world):
        tb, toff = gen.text(gen.SEED_WC + r, cap_bytes=20_000)
        words = oracle.wc(tb, toff)
        seg = g[r * stride: r * stride + int(counts[r])]
        assert int(counts[r]) == len(words) - 3
        for (w, c), row in zip(words, seg):
            assert row[0] == word_key(w) and row[1] == len(w) and row[2] == c and row[3] == r
            merged[w] = merged.get(w, 0) + c
    assert len(merged) > 100


def test_shard_range_covers():
    for n in (0, 1, 7, 1000):
        for world in (1, 2, 3, 8):
            rs = [merge.shard_range(n, r, world) for r in range(world)]
            assert rs[0][0] == 0 and rs[-1][1] == n
            assert all(rs[i][1] == rs[i + 1][0] for i in range(world - 1))
