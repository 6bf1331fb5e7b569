"""N>1 parity: bench.py's multi-rank path (torchrun, one process per GPU, each rank streaming its
contiguous shard through libbk on the GPU, then merge.py's collectives) must produce the SAME
result as the oracle over the whole data set (invariant I1: results independent of the GPU count,
PAPER.md P:29-31 independent segments).

Two ranks share cuda:0 over gloo (BK_BENCH_BACKEND=gloo: NCCL refuses two ranks on one device);
the GPU work and the merge kernels are the real ones, only the collectives' transport differs from
the 8-GPU NCCL run. Each rank dumps its merged result after the timed steps (bench.py --dump)."""
import os
import socket
import subprocess
import sys

import numpy as np
import pytest

import gen
import oracle
from paper_conf_ipps_mokhtaris14_b200 import bk

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
pytestmark = pytest.mark.gpu
WORLD = 2


def _port() -> int:
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def run_ranks(tmp_path, workload: str, gib: float, window_mib: int, extra=()) -> list[dict]:
    env = dict(os.environ, BK_BENCH_BACKEND="gloo")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", str(WORLD),
           "--master-addr", "127.0.0.1", "--master-port", str(_port()), "bench.py", "--gpus", str(WORLD),
           "--workload", workload, "--gib", str(gib), "--window-mib", str(window_mib), "--steps", "1",
           "--warmup", "3", "--no-cpu-baseline", "--no-dbuf", "--no-profile", "--dump", str(tmp_path), *extra]
    p = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=900)
    assert p.returncode == 0, p.stderr[-3000:]
    return [dict(np.load(tmp_path / f"rank{r}.npz")) for r in range(WORLD)]


def shards(workload: str, gib: float):
    sys.path.insert(0, ROOT)
    import bench
    bench.HUGE = None   # plain numpy pages, as the default bench run
    return [bench.make_shard(workload, gib, r, WORLD) for r in range(WORLD)]


def test_grep_two_ranks(tmp_path):
    res = run_ranks(tmp_path, "grep", 0.03, 8)
    sh = shards("grep", 0.03)
    total = int(res[0]["place"][1])
    glob = np.full(total, np.iinfo(np.uint64).max, np.uint64)
    for r in range(WORLD):
        off_, tot = (int(x) for x in res[r]["place"])
        assert tot == total
        glob[off_: off_ + len(res[r]["idx"])] = res[r]["idx"]
    # whole data set = the concatenated shards (rank r's records follow rank r-1's)
    buf = np.concatenate([s["buf"] for s in sh])
    offs = np.concatenate([sh[0]["off"], sh[1]["off"] + np.uint64(len(sh[0]["buf"]))])
    assert sh[1]["first"] == len(sh[0]["off"])
    want = oracle.grep(buf, offs, b"bigk")
    assert np.array_equal(glob, want) and total == len(want) > 0


def test_wordcount_two_ranks(tmp_path):
    res = run_ranks(tmp_path, "wordcount", 2 / 1024, 1)
    sh = shards("wordcount", 2 / 1024)
    rows = res[0]["rows"]
    assert np.array_equal(np.sort(rows, axis=0), np.sort(res[1]["rows"], axis=0))   # both ranks hold the merge
    got = sorted((sh[int(rk)]["buf"][int(o): int(o) + int(ln)].tobytes(), int(c))
                 for _, _, ln, c, rk, o in rows.astype(np.uint64))
    buf = np.concatenate([s["buf"] for s in sh])
    offs = np.concatenate([sh[0]["off"], sh[1]["off"] + np.uint64(len(sh[0]["buf"]))])
    assert got == oracle.wc(buf, offs)
    # the merged payload is the LOWEST rank's occurrence
    first_rank = {}
    for r in range(WORLD):
        for w, _ in oracle.wc(sh[r]["buf"], sh[r]["off"]):
            first_rank.setdefault(w, r)
    for _, _, ln, c, rk, o in rows.astype(np.uint64):
        assert first_rank[sh[int(rk)]["buf"][int(o): int(o) + int(ln)].tobytes()] == int(rk)


@pytest.mark.parametrize("workload", ["groupby", "groupby_sparse"])
def test_groupby_two_ranks(tmp_path, workload):
    gib = 0.03
    res = run_ranks(tmp_path, workload, gib, 8)
    sh = shards(workload, gib)
    stride = sh[0]["rec_size"]
    buf = np.concatenate([s["buf"] for s in sh])
    n = sum(s["n"] for s in sh)
    wc_, wq, wa = oracle.groupby(buf, n, stride, 4096)
    for r in range(WORLD):
        assert np.array_equal(res[r]["count"].astype(np.uint64), wc_)
        assert np.array_equal(res[r]["qty"].astype(np.uint64), wq)
        np.testing.assert_allclose(res[r]["amount"], wa, rtol=1e-5, atol=0)


def test_kmeans_two_ranks(tmp_path):
    gib = 0.01
    res = run_ranks(tmp_path, "kmeans", gib, 8)
    sh = shards("kmeans", gib)
    x = np.concatenate([s["buf"] for s in sh]).view(np.float32).reshape(-1, 16)
    wc_, ws, wchk, _ = oracle.kmeans(x, sh[0]["mu"])
    for r in range(WORLD):
        assert np.array_equal(res[r]["count"].astype(np.uint64), wc_)
        assert int(np.uint64(res[r]["chk"])) == wchk
        # |gpu - ref| <= 1e-5 * sum |x| per (cluster, dim): x > 0, so the sums bound it
        np.testing.assert_allclose(res[r]["sum"].reshape(ws.shape), ws, rtol=1e-5, atol=0)


def test_partition_two_ranks(tmp_path):
    gib = 0.02
    res = run_ranks(tmp_path, "partition", gib, 8)
    sh = shards("partition", gib)
    kv = np.concatenate([s["buf"] for s in sh]).view(np.uint64).reshape(-1, 2)
    wboff, wout = oracle.partition(kv, 1024)
    glob = np.zeros_like(wout)
    for r in range(WORLD):
        assert np.array_equal(res[r]["boff"].astype(np.uint64), wboff)
        # each rank's chunk-major runs placed at its global bucket offsets (merge_partition_offsets)
        bk.partition_materialize(res[r]["out"], res[r]["cc"], bucket_start=res[r]["start"], dst=glob)
    assert np.array_equal(glob, wout)


def test_kmer_two_ranks(tmp_path):
    gib = 0.005
    res = run_ranks(tmp_path, "kmer", gib, 8)
    sh = shards("kmer", gib)
    d = np.concatenate([s["buf"] for s in sh])
    n = sum(s["n"] for s in sh)
    okm, oct_ = oracle.kmer(d, n, k=31)
    rows = res[0]["rows"].astype(np.uint64)
    o = np.argsort(rows[:, 0])
    assert np.array_equal(rows[o, 0], okm) and np.array_equal(rows[o, 1], oct_)
