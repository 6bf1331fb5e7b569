#!/usr/bin/env python3
"""Table II on B200: bytes of explicit per-element addresses (the paper's
addrBuf, 8 B per accessed element) vs online-detected patterns, per workload, through
BK_K_PATTERN_STATS on the bench data sets; plus what sending them would cost on the measured
host link (8 B per address) relative to the data itself. Writes one JSON line per workload."""
import json
import sys

sys.path.insert(0, "/root/repo")
import numpy as np  # noqa: E402

import gen  # noqa: E402
from paper_conf_ipps_mokhtaris14_b200 import bk  # noqa: E402

LINK = 55.5e9
cases = []
tb, toff = gen.text(cap_bytes=64 << 20)
cases.append(("wordcount (1-B chars, whole lines)", tb, toff, 0, None, 1))
x = gen.points(n=1 << 24)
cases.append(("k-means (fp32 coordinates, 64-B points)", x.view(np.uint8).reshape(-1), None, 64, None, 4))
g = gen.groupby(n=1 << 24, stride=64)
cases.append(("group-by sparse (16 of 64 B, 4-B words)", g, None, 64, [(0, 16)], 4))
gb, goff = gen.grep_records(max_bytes=1 << 30)
cases.append(("grep (32-B key in variable records, 4-B words)", gb, goff, 0, [(16, 32)], 4))
for name, buf, off, rs, ext, elem in cases:
    n = len(off) if off is not None else len(buf) // rs
    with bk.Context(window_bytes=256 << 20, gather_mode="zc", record_size=rs) as ctx:
        ctx.register(buf, off, n_records=n)
        tot, _ = ctx.pattern_stats(ext, elem_bytes=elem, T=8)
        st = ctx.stats()
    accessed = tot["n_addresses"] * elem   # every accessed byte is covered by exactly one element address
    line = dict(workload=name, elem_bytes=elem, lanes=tot["n_lanes"], pattern_lanes=tot["n_pattern_lanes"],
                addresses=tot["n_addresses"], address_bytes=tot["address_bytes"], pattern_bytes=tot["pattern_bytes"],
                accessed_bytes=accessed,
                link_time_data_ms=accessed / LINK * 1e3,
                link_time_with_addresses_ms=(accessed + tot["address_bytes"]) / LINK * 1e3,
                link_time_with_patterns_ms=(accessed + tot["pattern_bytes"]) / LINK * 1e3)
    line["gain_patterns_vs_addresses"] = 1 - line["link_time_with_patterns_ms"] / line["link_time_with_addresses_ms"]
    print(json.dumps(line), flush=True)
