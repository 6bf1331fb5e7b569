"""Multi-GPU sharding and the final merge of per-GPU results.

Records are independent segments, so rank r streams its own contiguous record
range over its own host link with no data-path collective; the only exchange is this merge, run
once after the last chunk over torch.distributed (NCCL over NVLink on the GPU box, gloo in the
CPU tests). Every function here is plumbing around results libbk computed on the GPU:
  * aggregates (group-by, k-means) are written by bk_run straight into device tensors and
    all-reduced in place (no host round trip);
  * count tables (word count, k-mers) are all-gathered as compacted u64 rows and merged by key on
    the GPU by libbk's bk_merge_counts;
  * ordered outputs (grep indices, partition runs) need only their global offsets (all-gather of
    per-rank counts).
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
    """Group-by / k-means aggregates: element-wise sum over ranks, in place (u64 counts as int64
    wrap exactly; fp64 sums). gloo (CPU tests, ranks sharing one GPU) reduces a host copy."""
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


def gather_rows(rows: torch.Tensor, n: int) -> tuple[torch.Tensor, np.ndarray, int]:
    """All-gather every rank's first n rows of `rows` ([cap, W] int64, device) into one
    [world * stride, W] device tensor (segment r = rank r's rows, padded to the longest).
    Returns (gathered, per-rank row counts, stride)."""
    world = dist.get_world_size()
    dev = rows.device
    cnt = torch.tensor([n], dtype=torch.int64, device=_dev())
    allc = torch.empty(world, dtype=torch.int64, device=_dev())
    dist.all_gather_into_tensor(allc, cnt)
    counts = allc.cpu().numpy().astype(np.uint64)
    stride = max(int(counts.max()), 1)
    W = rows.shape[1]
    mine = rows[:stride] if rows.shape[0] >= stride else torch.cat(
        [rows, torch.zeros(stride - rows.shape[0], W, dtype=rows.dtype, device=dev)])
    mine = mine.contiguous()
    if dist.get_backend() == "nccl":
        out = torch.empty(world * stride, W, dtype=rows.dtype, device=dev)
        dist.all_gather_into_tensor(out, mine)
    else:   # gloo (CPU tests, ranks sharing one GPU): gather host copies
        parts = [torch.empty(stride, W, dtype=rows.dtype) for _ in range(world)]
        dist.all_gather(parts, mine.cpu())
        out = torch.cat(parts).to(dev)
    return out, counts, stride


def merge_count_rows(ctx, rows: torch.Tensor, n: int, key_u64: int, count_col: int,
                     cap: int | None = None) -> torch.Tensor:
    """Count tables: all-gather the compacted rows ([>= n, W] int64, device) of every rank, then
    merge them by key on this rank's GPU (libbk bk_merge_counts): one row per distinct key with the
    counts summed and the other words taken from the lowest rank's row. Returns the merged rows."""
    g, counts, stride = gather_rows(rows, n)
    W = rows.shape[1]
    cap = cap if cap is not None else int(counts.sum())
    out = torch.empty(max(cap, 1), W, dtype=torch.int64, device=rows.device)
    m = ctx.merge_counts(g, counts, stride, W, key_u64, count_col, out)
    return out[:m]


# row layouts of the count tables (u64 words; the key first)
WC_ROW = ("h1", "h2", "len", "count", "rank", "off")   # key = (h1, h2, len): the word's identity


def wordcount_rows(off, ln, cnt, h1, h2, rank: int) -> torch.Tensor:
    """Compacted word-count table of one rank (device tensors from Context.wordcount with hashes)
    as [n, 6] int64 rows in WC_ROW order."""
    n = off.shape[0]
    rk = torch.full((n,), rank, dtype=torch.int64, device=off.device)
    return torch.stack([h1.view(torch.int64), h2.view(torch.int64), ln.to(torch.int64),
                        cnt.view(torch.int64), rk, off.view(torch.int64)], dim=1).contiguous()


def merge_wordcount(ctx, off, ln, cnt, h1, h2) -> torch.Tensor:
    """Word count: all-gather of the compacted per-rank tables {h1, h2, len,
    count, rank, first_off}, merged by (h1, h2, len) on the GPU. A merged row's (rank, off) locates
    one occurrence of the word in that rank's shard."""
    rows = wordcount_rows(off, ln, cnt, h1, h2, dist.get_rank())
    return merge_count_rows(ctx, rows, rows.shape[0], key_u64=3, count_col=3)


def merge_kmer(ctx, km, ct) -> torch.Tensor:
    """k-mer tables (f4): rows {kmer, count}, merged by kmer."""
    rows = torch.stack([km.view(torch.int64), ct.view(torch.int64)], dim=1).contiguous()
    return merge_count_rows(ctx, rows, rows.shape[0], key_u64=1, count_col=1)
