"""Where does a word-count step's time go? wall (Python call) vs bk_run host time (ms_run) vs device
time (ms_device: compute-stream events around the run) vs the traced device span (CUPTI)."""
import sys, time
import numpy as np
sys.path.insert(0, ".")
import gen
from paper_conf_ipps_mokhtaris14_b200 import bk

buf, off = gen.text(gen.SEED_WC, cap_bytes=64 << 20)
cap = 1 << 20
out = (np.zeros(cap, np.uint64), np.zeros(cap, np.uint32), np.zeros(cap, np.uint64), np.zeros(cap, np.uint64),
       np.zeros(cap, np.uint64))
for trace in (False, True):
    ctx = bk.Context(device=0, window_bytes=8 << 20, keep_outputs_pinned=True, trace=trace)
    ctx.register(buf, off, n_records=len(off))
    wall, run, dev, span = [], [], [], []
    for i in range(40):
        t0 = time.perf_counter()
        ctx.wordcount(out=out)
        wall.append((time.perf_counter() - t0) * 1e3)
        s = ctx.stats()
        run.append(s["ms_run"]); dev.append(s["ms_device"]); span.append(s.get("ms_trace_span", 0.0))
    med = lambda v: float(np.median(v[10:]))
    print(f"trace={trace}: wall {med(wall):.3f} ms  bk_run {med(run):.3f} ms  device {med(dev):.3f} ms  "
          f"span {med(span):.3f} ms  -> {len(buf) / 1e6 / med(wall):.1f} GB/s wall (text only)")
    ctx.close()
