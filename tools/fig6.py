#!/usr/bin/env python3
"""Fig. 6-style stage breakdown on B200 (time of each pipeline stage, and
"address generation ... usually less than 20% of the slowest stage") from the committed
bench lines (profiles/r01_bench_*.json, per-stage busy sums of the profiled pass).

    python tools/fig6.py > profiles/r01_fig6.md
"""
import json
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
print("# Stage breakdown per step on B200 (Fig. 6 structure), from `profiles/r01_bench_*.json`\n")
print("Busy time of each stage summed over the step's chunks (profiled eager pass; stages of different "
      "chunks overlap, so the sums exceed the step). Transfer = DMA copies + zero-copy gathers "
      "(stages 2+3 fused) + write-back; assembly = host packing (CPU/HYBRID chunks, wall) + HBM->HBM "
      "interleave.\n")
print("| workload | gather | address generation ms | assembly ms (host / HBM) | transfer ms (DMA / ZC / D2H) | "
      "compute ms | slowest stage | addr-gen / slowest |")
print("|---|---|---|---|---|---|---|---|")
for w in ("grep", "groupby", "groupby_sparse", "kmeans", "partition", "wordcount", "kmer"):
    p = os.path.join(ROOT, "profiles", f"r01_bench_{w}.json")
    if not os.path.exists(p):
        continue
    d = json.load(open(p))
    st = d["stages_ms_per_step"]
    ag = st["ms_addrgen"]
    host, relay = st["ms_cpu_gather"], st["ms_relayout"]
    h2d, zc, d2h = st["ms_h2d"], st["ms_zc"], st.get("ms_d2h", 0.0)
    comp = st["ms_compute"]
    stages = {"assembly": host + relay, "transfer": h2d + zc + d2h, "compute": comp}
    slow = max(stages, key=stages.get)
    print(f"| {w} | {d['config']['gather_mode']} | {ag:.2f} | {host:.1f} / {relay:.1f} | {h2d:.1f} / {zc:.1f} / "
          f"{d2h:.1f} | {comp:.1f} | {slow} ({stages[slow]:.1f}) | {ag / stages[slow]:.1%} |")
print("\nThe paper's address-generation observation holds on B200 for every workload except word count, "
      "whose stage 1 reads each chunk's offsets zero-copy (one thread per record) and, at 0.44-MB chunks, is "
      "launch- and latency-dominated (these are eager-pass sums). On double-buffered descriptors it runs "
      "alongside the slot's previous compute; issuing it a whole ring earlier on its own streams (gated "
      "only by the compute that last used its descriptor set) was measured at 32.1 vs 33.3 GB/s "
      "(`tools/gpu_lookahead.sh`, reverted), so it does not hold the step back.")
