"""The bench's N>1 path (one process per GPU, torchrun launch, max-over-ranks timing, the merge
collectives of merge.py) end to end on ONE GPU: two ranks share cuda:0 over gloo
(BK_BENCH_BACKEND=gloo; NCCL refuses two ranks on one device). Every rank runs the real CUDA path;
only the collectives' transport differs from the 8-GPU NCCL run."""
import json
import os
import socket
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port() -> int:
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _run(args: list[str]) -> dict:
    env = dict(os.environ, BK_BENCH_BACKEND="gloo")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2", "--master-addr",
           "127.0.0.1", "--master-port", str(_port()), "bench.py", "--gpus", "2", *args]
    p = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=600)
    assert p.returncode == 0, p.stderr[-3000:]
    lines = [l for l in p.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, p.stdout[-2000:]   # rank 0 alone prints
    return json.loads(lines[0])


@pytest.mark.gpu
@pytest.mark.parametrize("workload,gib,window", [("grep", 0.25, 64), ("kmeans", 0.25, 64), ("wordcount", 1 / 64, 2),
                                                  ("partition", 0.125, 64), ("groupby", 0.25, 64)])
def test_bench_two_ranks(workload, gib, window):
    d = _run(["--workload", workload, "--gib", str(gib), "--window-mib", str(window), "--steps", "2", "--warmup", "3",
              "--no-cpu-baseline", "--no-dbuf"])
    assert d["n_gpus"] == 2 and d["steps"] == 2 and d["scaling"] == "weak"
    assert d["value"] > 0 and d["e2e"]["value"] > 0 and d["gpu_launches"] > 0
    assert d["config"]["bytes_per_gpu"] > 0 and d["config"]["parallelism"] == "dp2 (contiguous record shards, one PCIe link per GPU)"


@pytest.mark.gpu
def test_reference_arm_two_ranks():
    d = _run(["--impl", "reference", "--workload", "groupby", "--gib", "0.05", "--steps", "1", "--warmup", "3"])
    assert d["impl"] == "reference" and d["value"] > 0 and d["cpu_baseline"]["kind"] == "oracle"
