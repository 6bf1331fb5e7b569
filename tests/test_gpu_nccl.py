"""The NCCL code path of the multi-GPU merge, executed on a one-GPU box: bench.py under
`torchrun --nproc-per-node 1` with BK_BENCH_DIST=1 initialises an NCCL process group at world size 1
and takes the distributed path end to end — results written by bk_run into device tensors, the
merge.py collectives as NCCL calls on them (all_reduce in place, all_gather_into_tensor of counts and
of the compacted count-table rows), the GPU merge of the gathered rows (bk_merge_counts), the
max-over-ranks timing all-reduce. NCCL refuses two ranks on one device, so this is the only way one
GPU runs those calls; the two-rank arithmetic of the merge is covered by test_gpu_ranks_parity.py
(gloo transport). Results must equal the oracle over the shard."""
import os
import socket
import subprocess
import sys

import numpy as np
import pytest

import oracle
from paper_conf_ipps_mokhtaris14_b200 import bk

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
pytestmark = pytest.mark.gpu


def _port() -> int:
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def run_nccl(tmp_path, workload: str, gib: float, window_mib: int) -> tuple[dict, str]:
    env = dict(os.environ, BK_BENCH_DIST="1", BK_BENCH_BACKEND="nccl")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "1",
           "--master-addr", "127.0.0.1", "--master-port", str(_port()), "bench.py", "--gpus", "1",
           "--workload", workload, "--gib", str(gib), "--window-mib", str(window_mib), "--steps", "1",
           "--warmup", "3", "--no-cpu-baseline", "--no-dbuf", "--no-profile", "--no-trace", "--dump", str(tmp_path)]
    p = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=900)
    assert p.returncode == 0, p.stderr[-3000:]
    return dict(np.load(tmp_path / "rank0.npz")), p.stdout


def shard(workload: str, gib: float) -> dict:
    sys.path.insert(0, ROOT)
    import bench
    bench.HUGE = None
    return bench.make_shard(workload, gib, 0, 1)


def test_nccl_grep(tmp_path):
    res, out = run_nccl(tmp_path, "grep", 0.02, 8)
    sh = shard("grep", 0.02)
    want = oracle.grep(sh["buf"], sh["off"], b"bigk")
    assert tuple(int(x) for x in res["place"]) == (0, len(want)) and len(want) > 0
    assert np.array_equal(res["idx"], want)
    assert '"n_gpus": 1' in out


def test_nccl_wordcount(tmp_path):
    res, _ = run_nccl(tmp_path, "wordcount", 2 / 1024, 1)
    sh = shard("wordcount", 2 / 1024)
    rows = res["rows"].astype(np.uint64)
    assert (rows[:, 4] == 0).all()   # rank column
    got = sorted((sh["buf"][int(o): int(o) + int(ln)].tobytes(), int(c)) for _, _, ln, c, _, o in rows)
    assert got == oracle.wc(sh["buf"], sh["off"])


@pytest.mark.parametrize("workload", ["groupby", "groupby_sparse"])
def test_nccl_groupby(tmp_path, workload):
    res, _ = run_nccl(tmp_path, workload, 0.02, 8)
    sh = shard(workload, 0.02)
    wc_, wq, wa = oracle.groupby(sh["buf"], sh["n"], sh["rec_size"], 4096)
    assert np.array_equal(res["count"].astype(np.uint64), wc_)
    assert np.array_equal(res["qty"].astype(np.uint64), wq)
    np.testing.assert_allclose(res["amount"], wa, rtol=1e-5, atol=0)


def test_nccl_kmeans(tmp_path):
    res, _ = run_nccl(tmp_path, "kmeans", 0.01, 8)
    sh = shard("kmeans", 0.01)
    x = sh["buf"].view(np.float32).reshape(-1, 16)
    wc_, ws, wchk, _ = oracle.kmeans(x, sh["mu"])
    assert np.array_equal(res["count"].astype(np.uint64), wc_)
    assert int(np.uint64(res["chk"])) == wchk
    np.testing.assert_allclose(res["sum"].reshape(ws.shape), ws, rtol=1e-5, atol=0)


def test_nccl_partition(tmp_path):
    res, _ = run_nccl(tmp_path, "partition", 0.02, 8)
    sh = shard("partition", 0.02)
    kv = sh["buf"].view(np.uint64).reshape(-1, 2)
    wboff, wout = oracle.partition(kv, 1024)
    assert np.array_equal(res["boff"].astype(np.uint64), wboff)
    glob = np.zeros_like(wout)
    bk.partition_materialize(res["out"], res["cc"], bucket_start=res["start"], dst=glob)
    assert np.array_equal(glob, wout)


def test_nccl_kmer(tmp_path):
    res, _ = run_nccl(tmp_path, "kmer", 0.005, 8)
    sh = shard("kmer", 0.005)
    okm, oct_ = oracle.kmer(sh["buf"], sh["n"], k=31)
    rows = res["rows"].astype(np.uint64)
    o = np.argsort(rows[:, 0])
    assert np.array_equal(rows[o, 0], okm) and np.array_equal(rows[o, 1], oct_)
