"""Where does a word-count step's time go? wall (Python call) vs bk_run host time vs device time."""
import sys, time
import numpy as np
sys.path.insert(0, ".")
import gen
from paper_conf_ipps_mokhtaris14_b200 import bk

buf, off = gen.text(gen.SEED_WC, cap_bytes=64 << 20)
ctx = bk.Context(device=0, window_bytes=8 << 20, n_slots=int(sys.argv[1]) if len(sys.argv) > 1 else 4)
ctx.register(buf, off, n_records=len(off))
out = (np.zeros(1 << 20, np.uint64), np.zeros(1 << 20, np.uint32), np.zeros(1 << 20, np.uint64))
for reuse in (False, True):
    wall, run, dev = [], [], []
    for i in range(30):
        t0 = time.perf_counter()
        ctx.wordcount(out=out if reuse else None)
        wall.append((time.perf_counter() - t0) * 1e3)
        s = ctx.stats()
        run.append(s["ms_run"]); dev.append(s["ms_device"])
    print(f"reuse_out={reuse}: wall {np.median(wall[5:]):.3f} ms  bk_run {np.median(run[5:]):.3f} ms  "
          f"device {np.median(dev[5:]):.3f} ms  -> {64 * 1.048576 / np.median(wall[5:]):.1f} GB/s wall")
ctx.close()
