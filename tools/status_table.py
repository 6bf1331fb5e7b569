#!/usr/bin/env python3
"""DESIGN.md §9 / README status rows from the committed bench lines (profiles/<round>_bench_*.json).

    python tools/status_table.py design [r02]   # the §9 table rows
    python tools/status_table.py readme [r02]   # the README table rows
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
ROWS = [
    ("grep", "C2 grep 16 GiB (default bench)", "Grep, 16 GiB", "host packing + zero-copy request rate"),
    ("groupby", "C5 group-by 16 GiB dense", "Group-by, 16 GiB", ""),
    ("groupby32", "C5 group-by 32 GiB dense (C5's per-GPU share at 8 GPUs)", "Group-by, 32 GiB", ""),
    ("groupby_sparse", "C5 group-by sparse 16 GiB (64-B records, 25% read)", "Group-by sparse (25% read), 16 GiB", ""),
    ("kmeans", "C3 k-means 16 GiB, K=64", "K-means, 16 GiB", ""),
    ("kmeans256", "C3 k-means 16 GiB, K=256", "K-means K=256, 16 GiB", ""),
    ("partition", "C4 partition 8 GiB, 1024 buckets (D2H out)", "Partition, 8 GiB", ""),
    ("wordcount", "C1 word count 64 MiB, 8 MiB window", "Word count, 64 MiB (8 MiB window)", ""),
    ("kmer", "f4 k-mers 4 GiB (k = 31)", "k-mers, 4 GiB", ""),
]


RND = sys.argv[2] if len(sys.argv) > 2 else "r01"


def load(w, rnd=None):
    p = os.path.join(ROOT, "profiles", f"{rnd or RND}_bench_{w}.json")
    return json.load(open(p)) if os.path.exists(p) else None


def roof(d):
    """the dominant stage's roofline fraction and its bound"""
    r = d.get("roofline") or {}
    k = r.get("kernel", "")
    what = ("fused kernel" if "fused" in k else "ZC gather" if "zero-copy" in k else "H2D DMA" if "H2D" in k else
            "D2H DMA" if "D2H" in k else "compute")
    s = f"{r.get('frac', float('nan')):.2f} ({what})"
    hs = r.get("hybrid_schedule")
    if hs:
        s += f"; link+host schedule {hs['frac']:.2f}"
    return s


def prev(w):
    """the same line in round 1, when it exists"""
    d = load(w, "r01") if RND != "r01" else None
    if d is None:
        return "—"
    fd = d.get("link_full_duplex")
    return f"{d['value']:.1f}" + (" each way" if fd else "")


def overlap(d):
    """copy/compute overlap of the timed (graph-replayed) pass when traced, else the profiled pass"""
    t = d.get("timed_pass_trace")
    if d["config"].get("gather_mode") == "fused":
        return "one launch"
    if t and t.get("compute_busy_ms"):
        return f"{t['overlap_frac']:.2f}"
    return f"{d['overlap']['overlap_frac']:.2f}"


def gbs(v):
    return f"{v:.1f} GB/s" if v >= 1 else f"{v:.2g} GB/s"


def design():
    for w, name, _, _ in ROWS:
        d = load(w)
        if d is None:
            continue
        fd = d.get("link_full_duplex")
        val = f"{d['value']:.1f} each way" if fd else f"{d['value']:.1f}"
        frac = (f"{d['link']['frac']:.2f} (H2D); {fd['frac']:.2f} of the {fd['peak_each_way_gbs']:.1f} GB/s "
                f"bidirectional per-direction peak") if fd else f"{d['link']['frac']:.2f}"
        db = d.get("baseline_dbuf")
        dbs = f"{db['bigkernel_speedup']:.2f}× ({db['value']:.1f})" if db else "—"
        mt = d.get("cpu_mt_baseline")
        cb = d.get("cpu_baseline") or {}
        print(f"| {name} | {d['config']['gather_mode'].upper()} | {val} | {prev(w)} | {d['ms_per_step']:.3g} | {frac} | "
              f"{roof(d)} | {overlap(d)} | {dbs} | {gbs(mt['value']) if mt else '—'} | "
              f"{gbs(cb['value']) if cb.get('value') else '—'} |")


def readme():
    for w, _, name, note in ROWS:
        d = load(w)
        if d is None:
            continue
        fd = d.get("link_full_duplex")
        val = f"{d['value']:.1f} each way" if fd else f"{d['value']:.1f}"
        frac = f"{fd['frac']:.2f} of bidirectional" if fd else f"{d['link']['frac']:.2f}" + (f" ({note})" if note else "")
        db = d.get("baseline_dbuf")
        sp = f"{db['bigkernel_speedup']:.2f}×" if db else "—"
        print(f"| {name} | {val} | {frac} | {sp} |")


if __name__ == "__main__":
    {"design": design, "readme": readme}[sys.argv[1] if len(sys.argv) > 1 else "design"]()
