"""Does cudaHostRegister accept gen.alloc mappings (THP / 4K) on this box? Not product code."""
import sys, time
sys.path.insert(0, "/root/repo")
import numpy as np, torch, gen
cr = torch.cuda.cudart()
for huge, size, flags in ((True, 1 << 30, 3), (True, 16 << 30, 0), (True, 16 << 30, 3), (False, 16 << 30, 3), (True, (16 << 30) - 4000, 3)):
    a = gen.alloc(size, huge=huge)
    a[::4096] = 7
    t0 = time.time()
    r = cr.cudaHostRegister(a.ctypes.data, size, flags)
    print("huge", huge, "size", size, "flags", flags, "ret", r, "t", round(time.time() - t0, 3), flush=True)
    if int(r) == 0:
        cr.cudaHostUnregister(a.ctypes.data)
    del a
print(open("/proc/meminfo").read().split("AnonHugePages:")[1].split("\n")[0])
