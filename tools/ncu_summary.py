#!/usr/bin/env python3
"""Summarise ncu output for profiles/: a launch list (gpu__time_duration per launch) grouped by
kernel with each kernel's share, and key metrics of a --set full capture.

    python tools/ncu_summary.py launches gpurun_out/r01_launches_grep.csv
    python tools/ncu_summary.py full gpurun_out/r01_prof_grep.ncu-rep
"""
import csv
import io
import re
import subprocess
import sys
from collections import defaultdict

FULL_METRICS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread", "launch__grid_size",
    "launch__block_size", "pcie__read_bytes.sum.per_second", "pcie__write_bytes.sum.per_second",
    "syslts__t_sectors_srcunit_tex_aperture_sysmem_op_read_lookup_miss.sum",
    "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum", "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum",
    "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio", "smsp__inst_executed.sum",
]


def short(name: str) -> str:
    name = re.sub(r"\(.*", "", name)
    return name.replace("void ", "").replace("(anonymous namespace)::", "").replace("unnamed>::", "").strip()


def launches(path: str) -> None:
    text = open(path).read()
    start = text.find('"ID"')
    rows = list(csv.reader(io.StringIO(text[start:])))
    hdr = rows[0]
    ki, mi, vi = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value")
    agg = defaultdict(lambda: [0, 0.0])
    for r in rows[1:]:
        if len(r) <= vi or r[mi] != "gpu__time_duration.sum":
            continue
        v = float(r[vi].replace(",", ""))
        unit = r[hdr.index("Metric Unit")] if "Metric Unit" in hdr else "ns"
        ns = v * {"ns": 1, "usecond": 1e3, "us": 1e3, "msecond": 1e6, "ms": 1e6, "nsecond": 1}.get(unit, 1)
        k = short(r[ki])
        agg[k][0] += 1
        agg[k][1] += ns
    tot = sum(v[1] for v in agg.values())
    print(f"# launch list: {path}  (ncu gpu__time_duration, --clock-control none; serialised, cold-cache)")
    print(f"# total {sum(v[0] for v in agg.values())} launches, {tot / 1e6:.3f} ms summed device time")
    print("| kernel | launches | total ms | mean us | share |")
    print("|---|---:|---:|---:|---:|")
    for k, (n, ns) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        print(f"| {k} | {n} | {ns / 1e6:.3f} | {ns / n / 1e3:.1f} | {ns / tot:.1%} |")


def full(path: str) -> None:
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    print(f"# ncu --set full summary: {path}")
    for r in rows[2:]:
        print(f"\n## {short(r[hdr.index('Kernel Name')])}")
        for m in FULL_METRICS:
            if m in hdr:
                i = hdr.index(m)
                print(f"- {m} = {r[i]} {units[i]}")


if __name__ == "__main__":
    {"launches": launches, "full": full}[sys.argv[1]](sys.argv[2])
