"""Small out-of-core runs of every kernel and gather mode, for compute-sanitizer (SURVEY §4:
memcheck / racecheck / synccheck with tiny windows so many chunks and slot reuse occur)."""
import sys

sys.path.insert(0, "/root/repo")
import numpy as np  # noqa: E402

import gen  # noqa: E402
from paper_conf_ipps_mokhtaris14_b200 import bk  # noqa: E402

buf, off = gen.text(cap_bytes=1 << 19)
for mode in ("zc", "dense", "cpu"):
    with bk.Context(window_bytes=96 << 10, n_slots=3, gather_mode=mode, no_graph=True) as ctx:
        ctx.register(buf, off)
        ctx.wordcount(cap=1 << 16)
gb, goff = gen.grep_records(n=20000)
for mode in ("zc", "hybrid"):
    with bk.Context(window_bytes=256 << 10, n_slots=3, gather_mode=mode) as ctx:
        ctx.register(gb, goff)
        ctx.grep(b"bigk", cap=20000)
g = gen.groupby(n=100_000, stride=64)
with bk.Context(window_bytes=512 << 10, record_size=64) as ctx:
    ctx.register(g, None, n_records=100_000)
    ctx.groupby(4096)
x = gen.points(n=50_000)
with bk.Context(window_bytes=512 << 10, record_size=64) as ctx:
    ctx.register(x.view(np.uint8).reshape(-1), None, n_records=50_000)
    ctx.kmeans(x[:64], cid=np.empty(50_000, np.int32))
kv = gen.kv(n=100_000)
with bk.Context(window_bytes=1 << 20, record_size=16) as ctx:
    ctx.register(kv.view(np.uint8).reshape(-1), None, n_records=100_000)
    ctx.partition(1024)
# later round-1 paths: ZC per-slot staging streams + double-buffered descriptors (graph and eager),
# host-packed CPU chunks with the GPU interleave, order-independent grep, k-mers, online patterns
for ng in (False, True):
    with bk.Context(window_bytes=128 << 10, n_slots=4, gather_mode="zc", no_graph=ng) as ctx:
        ctx.register(buf, off)
        ctx.wordcount(cap=1 << 16)
        ctx.wordcount(cap=1 << 16)
for mode in ("cpu", "dense"):
    with bk.Context(window_bytes=256 << 10, n_slots=3, gather_mode=mode) as ctx:
        ctx.register(gb, goff)
        ctx.grep(b"bigk", cap=20000)
for mode in ("cpu", "hybrid"):
    with bk.Context(window_bytes=512 << 10, record_size=64, gather_mode=mode) as ctx:
        ctx.register(g, None, n_records=100_000)
        ctx.groupby(4096)
d = gen.dna(n=20_000, genome_len=1 << 16, err_pm=2, n_pm=3)
for mode in ("hybrid", "zc", "cpu"):
    with bk.Context(window_bytes=1 << 20, record_size=256, gather_mode=mode) as ctx:
        ctx.register(d, None, n_records=20_000)
        ctx.kmer(k=31, table_slots=1 << 22)
with bk.Context(window_bytes=256 << 10) as ctx:
    ctx.register(buf, off)
    ctx.pattern_stats(elem_bytes=1, T=8)
print("sanitize run done")
# TMA-staged stage 4 (dense / cpu), grep masks with long lanes, G = 8192 tables, k-means dbuf baseline
g16 = gen.groupby(n=200_000, G=8192)
for mode in ("dense", "cpu", "zc"):
    with bk.Context(window_bytes=1 << 20, record_size=16, gather_mode=mode) as ctx:
        ctx.register(g16, None, n_records=200_000)
        ctx.groupby(8192)
for mode in ("cpu", "zc"):
    with bk.Context(window_bytes=1 << 20, gather_mode=mode, lane_bytes=4096) as ctx:
        ctx.register(gb, goff)
        ctx.grep(b"a", cap=20000)
with bk.Context(window_bytes=512 << 10, record_size=64, baseline_dbuf=True) as ctx:
    ctx.register(x.view(np.uint8).reshape(-1), None, n_records=50_000)
    ctx.kmeans(x[:7])
# late round 1: profiled runs (nested write-back D2H events), tiny / ragged data sets, user kernels
with bk.Context(window_bytes=512 << 10, record_size=64, profile=True) as ctx:
    ctx.register(x.view(np.uint8).reshape(-1), None, n_records=50_000)
    ctx.kmeans(x[:64], cid=np.empty(50_000, np.int32))
with bk.Context(window_bytes=1 << 20, record_size=16, profile=True) as ctx:
    ctx.register(kv.view(np.uint8).reshape(-1), None, n_records=100_000)
    ctx.partition(256)
for n in (1, 33):
    for mode in ("zc", "cpu", "dense", "hybrid"):
        tb, to = gen.text(cap_recs=n)
        with bk.Context(window_bytes=1 << 20, gather_mode=mode) as ctx:
            ctx.register(tb, to[:n])
            ctx.wordcount(cap=1 << 10)
        eb, eo = gen.grep_records(n=n)
        with bk.Context(window_bytes=1 << 20, gather_mode=mode) as ctx:
            ctx.register(eb, eo)
            ctx.grep(b"", cap=n)
        with bk.Context(window_bytes=1 << 20, record_size=16, gather_mode=mode) as ctx:
            ctx.register(kv[:n].view(np.uint8).reshape(-1), None, n_records=n)
            if mode != "hybrid":
                ctx.partition(64)
print("sanitize run ok")
# round 2: the fused single-launch word count (zero-copy loaders and the copy-engine feed), address
# mode (patterns / explicit) incl. a layout dump, the GPU merge of count tables, two-phase k-mers
import os  # noqa: E402
for feed in ("zc", "dma"):
    os.environ["BK_FUSED_FEED"] = feed
    with bk.Context(window_bytes=256 << 10) as ctx:
        ctx.register(buf, off)
        ctx.wordcount(cap=1 << 16)
        ctx.wordcount(cap=1 << 16)
os.environ.pop("BK_FUSED_FEED")
for nop in (False, True):
    with bk.Context(window_bytes=512 << 10, gather_mode="addr", no_patterns=nop) as ctx:
        ctx.register(buf, off)
        ctx.wordcount(cap=1 << 16)
        ctx.layout_dump(1)
    with bk.Context(window_bytes=512 << 10, record_size=64, gather_mode="addr", no_patterns=nop) as ctx:
        ctx.register(g, None, n_records=100_000)
        ctx.groupby(4096)
import torch  # noqa: E402
rows = torch.randint(0, 1 << 20, (3 * 4096, 6), dtype=torch.int64, device="cuda")
out = torch.empty(3 * 4096, 6, dtype=torch.int64, device="cuda")
with bk.Context(window_bytes=1 << 20) as ctx:
    ctx.merge_counts(rows, [4096, 100, 4000], 4096, 6, 3, 3, out)
with bk.Context(window_bytes=1 << 20, record_size=256, gather_mode="zc") as ctx:
    ctx.register(d, None, n_records=20_000)
    ctx.kmer(k=31, table_slots=1 << 20)
    ctx.kmer(k=31, table_slots=1 << 22)
# results stored by the final kernels straight into kept-pinned host arrays (mapped) and device tensors;
# a mid-run flush
import numpy as np  # noqa: E402
os.environ["BK_KMER_F"] = "1"
with bk.Context(window_bytes=1 << 20, record_size=256, keep_outputs_pinned=True) as ctx:
    ctx.register(d, None, n_records=20_000)
    kout = (np.zeros(1 << 20, np.uint64), np.zeros(1 << 20, np.uint64))
    ctx.kmer(k=31, table_slots=1 << 22, out=kout)
    ctx.kmer(k=31, table_slots=1 << 22, out=(torch.zeros(1 << 20, dtype=torch.int64, device="cuda"),
                                             torch.zeros(1 << 20, dtype=torch.int64, device="cuda")))
os.environ.pop("BK_KMER_F")
with bk.Context(window_bytes=256 << 10, keep_outputs_pinned=True) as ctx:
    ctx.register(buf, off)
    wout = (np.zeros(1 << 16, np.uint64), np.zeros(1 << 16, np.uint32), np.zeros(1 << 16, np.uint64))
    ctx.wordcount(out=wout)
    ctx.wordcount(out=wout)
print("sanitize run (round 2) done")
