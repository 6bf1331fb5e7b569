#!/usr/bin/env python3
"""Table II on B200, MEASURED (§IV.A): the paper's address mode
(BK_GATHER_ADDR) run end to end — GPU address generation, per-lane patterns or explicit addresses
written to pinned host memory, host assembly from them, DMA, the unchanged kernel — once with the
online pattern recogniser and once sending every element address (BK_FLAG_NO_PATTERNS), on the
same data, window and box. Reports per variant the device time per run, the address bytes the GPU
wrote to the host, the payload DMA'd, and the gain from patterns = 1 - t(patterns) / t(addresses)
(the paper's column), next to the product path (AUTO) for context. One JSON line per workload."""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402

import gen  # noqa: E402
from paper_conf_ipps_mokhtaris14_b200 import bk  # noqa: E402

RUNS = int(os.environ.get("T2_RUNS", "3"))


def run(ctxkw, reg, call):
    with bk.Context(**ctxkw) as ctx:
        reg(ctx)
        call(ctx)   # warm-up (plan, pinning of outputs)
        ts = []
        for _ in range(RUNS):
            t0 = time.perf_counter()
            call(ctx)
            ts.append(time.perf_counter() - t0)
        st = ctx.stats()
    return min(ts), st


def main():
    cases = []
    tb, toff = gen.text(cap_bytes=64 << 20)
    cases.append(("wordcount (C1 text, 1-B elements)", dict(window_bytes=256 << 20),
                  lambda c: c.register(tb, toff), lambda c: c.wordcount(cap=1 << 20), len(tb)))
    n = 1 << 24
    x = gen.points(n=n)
    mu = x[:64].copy()
    cases.append(("k-means (16 fp32 per 64-B point, 8-B elements)", dict(window_bytes=2 << 30, record_size=64),
                  lambda c: c.register(x.view(np.uint8).reshape(-1), None, n_records=n), lambda c: c.kmeans(mu),
                  n * 64))
    g = gen.groupby(n=n, stride=64)
    cases.append(("group-by sparse (16 of 64 B, 8-B elements)", dict(window_bytes=2 << 30, record_size=64),
                  lambda c: c.register(g, None, n_records=n), lambda c: c.groupby(4096), n * 64))
    gb, goff = gen.grep_records(max_bytes=1 << 30)
    idx = np.empty(len(goff), np.uint64)
    cases.append(("grep (32-B key in variable records, 8-B elements)", dict(window_bytes=2 << 30),
                  lambda c: c.register(gb, goff), lambda c: c.grep(b"bigk", out=idx), len(gb)))
    for name, kw, reg, call, nbytes in cases:
        res = {}
        for tag, extra in (("patterns", dict(gather_mode="addr")), ("addresses", dict(gather_mode="addr", no_patterns=True)),
                           ("product", dict())):
            t, st = run({**kw, **extra}, reg, call)
            res[tag] = dict(s=t, gbs=nbytes / t / 1e9, bytes_addr=st["bytes_addr"], bytes_h2d=st["bytes_h2d"] + st["bytes_meta"],
                            pattern_lanes=st["n_pattern_lanes"], lanes=st["n_addr_lanes"],
                            addresses=st["n_addresses"], explicit=st["n_explicit_addr"], elem=st["addr_elem_bytes"],
                            host_assembly_ms=st["ms_cpu_gather"], addr_wait_ms=st["ms_addr_wait"],
                            mode={1: "zc", 2: "cpu", 3: "dense", 4: "hybrid", 5: "fused", 6: "addr"}.get(st["gather_mode"]))
        line = dict(workload=name, bytes=nbytes, **res,
                    gain_patterns_vs_addresses=1 - res["patterns"]["s"] / res["addresses"]["s"])
        print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
