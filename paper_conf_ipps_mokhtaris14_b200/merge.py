"""Multi-GPU sharding and the final merge of per-GPU results.

Records are independent segments, so rank r streams its own contiguous record
range over its own host link with no data-path collective; the only exchange is this merge, run
once after the last chunk over torch.distributed (NCCL over NVLink on the GPU box, gloo in the
CPU tests). Every function here is plumbing around results libbk already computed on the GPU.
"""
from __future__ import annotations

import numpy as np
import torch
import torch.distributed as dist


def shard_range(n: int, rank: int, world: int) -> tuple[int, int]:
    """Contiguous, balanced record range [lo, hi) of rank r (fixed-length records)."""
    lo = n * rank // world
    hi = n * (rank + 1) // world
    return lo, hi


def _dev():
    return torch.device("cuda", torch.cuda.current_device()) if dist.get_backend() == "nccl" else torch.device("cpu")


def merge_sum(t: torch.Tensor) -> torch.Tensor:
    """Group-by / k-means aggregates: element-wise sum over ranks (counts and fp64 sums)."""
    if t.is_cuda and dist.get_backend() != "nccl":
        h = t.cpu()
        dist.all_reduce(h, op=dist.ReduceOp.SUM)
        t.copy_(h)
        return t
    dist.all_reduce(t, op=dist.ReduceOp.SUM)
    return t


def merge_checksum(chk: int) -> int:
    """k-means checksum: sum mod 2^64 over ranks (int64 all-reduce wraps)."""
    t = torch.tensor([np.uint64(chk).astype(np.int64)], dtype=torch.int64, device=_dev())
    dist.all_reduce(t)
    return int(np.int64(t.item()).astype(np.uint64))


def merge_grep_offsets(n_match: int) -> tuple[int, int]:
    """Grep: each rank's ascending index list lands after the lists of lower ranks (rank ranges
    ascend). Returns (this rank's global output offset, global match count)."""
    world, rank = dist.get_world_size(), dist.get_rank()
    mine = torch.tensor([n_match], dtype=torch.int64, device=_dev())
    allc = torch.empty(world, dtype=torch.int64, device=_dev())
    dist.all_gather_into_tensor(allc, mine)
    c = allc.cpu().numpy()
    return int(c[:rank].sum()), int(c.sum())


def merge_partition_offsets(bucket_count: np.ndarray) -> tuple[np.ndarray, np.ndarray]:
    """Partition: global bucket-major placement of each rank's runs. Returns (start[b] of this
    rank's records of bucket b in the final stable order, global bucket offsets boff[B+1])."""
    world, rank = dist.get_world_size(), dist.get_rank()
    B = len(bucket_count)
    mine = torch.from_numpy(bucket_count.astype(np.int64)).to(_dev())
    allc = torch.empty(world * B, dtype=torch.int64, device=_dev())
    dist.all_gather_into_tensor(allc, mine)
    c = allc.cpu().numpy().reshape(world, B)
    tot = c.sum(0)
    boff = np.concatenate([[0], np.cumsum(tot)]).astype(np.uint64)
    start = boff[:-1].astype(np.int64) + c[:rank].sum(0)
    return start.astype(np.uint64), boff


def merge_wordcount(words: dict[bytes, int]) -> dict[bytes, int]:
    """Word count: union of the per-rank (word -> count) tables; every rank gets the merged table."""
    world = dist.get_world_size()
    out: list = [None] * world
    dist.all_gather_object(out, words)
    merged: dict[bytes, int] = {}
    for d in out:
        for w, c in d.items():
            merged[w] = merged.get(w, 0) + c
    return merged
