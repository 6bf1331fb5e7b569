"""CPU oracle for the BigKernel hot path — TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference leg may
import this module. The product (paper_conf_ipps_mokhtaris14_b200) never imports it and shares
no code with it (oracle/oracle.c is plain single-threaded C; see oracle.h for the passages
each function follows). Parity status of every function: DESIGN.md §Oracle.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libbkoracle.so")
_SRC = os.path.join(_HERE, "oracle.c")
_lib = None


def build() -> str:
    if not os.path.exists(_SO) or os.path.getmtime(_SO) < max(os.path.getmtime(_SRC), os.path.getmtime(_SRC[:-1] + "h")):
        subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fPIC", "-shared", "-Wall", _SRC, "-o", _SO, "-lm"])
    return _SO


def lib():
    global _lib
    if _lib is None:
        l = C.CDLL(build())
        u64, u32, i64, p = C.c_uint64, C.c_uint32, C.c_int64, C.c_void_p
        l.oracle_wc.restype = i64
        l.oracle_wc.argtypes = [p, u64, p, u64, p, p, p, u64]
        l.oracle_grep.restype = i64
        l.oracle_grep.argtypes = [p, u64, p, u64, p, u32, u64, p, u64]
        l.oracle_kmeans.restype = None
        l.oracle_kmeans.argtypes = [p, u64, p, u32, u64, p, p, p, p]
        l.oracle_partition.restype = C.c_int
        l.oracle_partition.argtypes = [p, u64, u32, p, p]
        l.oracle_groupby.restype = C.c_int
        l.oracle_groupby.argtypes = [p, u64, u32, u32, p, p, p]
        l.oracle_plan_chunks.restype = i64
        l.oracle_plan_chunks.argtypes = [p, u64, u64, u64, u32, p, p, u64, p, u64]
        l.oracle_layout.restype = i64
        l.oracle_layout.argtypes = [p, p, u64, u64, u64, u32, p, p, u64, u64, u32, p, p, p, p, u64]
        l.oracle_pattern.restype = C.c_int
        l.oracle_pattern.argtypes = [p, u32, u32, p]
        l.oracle_kmer.restype = i64
        l.oracle_kmer.argtypes = [p, u64, u32, u32, u32, u32, p, p, u64]
        l.oracle_pattern_online.restype = C.c_int
        l.oracle_pattern_online.argtypes = [p, u64, u32, u32, p]
        _lib = l
    return _lib


def _p(a):
    if a is None:
        return None
    a = np.ascontiguousarray(a)
    return a.ctypes.data


def _u8(b) -> np.ndarray:
    if isinstance(b, (bytes, bytearray)):
        return np.frombuffer(bytes(b), np.uint8) if len(b) else np.zeros(1, np.uint8)[:0]
    return np.ascontiguousarray(b, dtype=np.uint8)


def wc(text, off) -> list[tuple[bytes, int]]:
    """O1: sorted [(word, count)]."""
    t = _u8(text)
    off = np.ascontiguousarray(off, np.uint64)
    tb = t if len(t) else np.zeros(1, np.uint8)
    cap = 1024
    while True:
        wo = np.empty(cap, np.uint64); wl = np.empty(cap, np.uint32); wcnt = np.empty(cap, np.uint64)
        V = lib().oracle_wc(_p(tb), len(t), _p(off) if len(off) else None, len(off), _p(wo), _p(wl), _p(wcnt), cap)
        if V >= 0:
            break
        cap = -V
    tbytes = t.tobytes()
    return [(tbytes[int(wo[i]): int(wo[i]) + int(wl[i])], int(wcnt[i])) for i in range(V)]


def grep(buf, off, pattern: bytes = b"bigk", first: int = 0) -> np.ndarray:
    """O2: ascending matching record indices (+first)."""
    b = _u8(buf)
    off = np.ascontiguousarray(off, np.uint64)
    pat = np.frombuffer(pattern, np.uint8) if pattern else np.zeros(1, np.uint8)
    cap = len(off)
    idx = np.empty(max(cap, 1), np.uint64)
    m = lib().oracle_grep(_p(b) if len(b) else None, len(b), _p(off) if len(off) else None, len(off),
                          _p(pat), len(pattern), first, _p(idx), cap)
    if m < 0:
        raise ValueError("record shorter than 48 bytes")
    return idx[:m].copy()


def kmeans(x, mu, first: int = 0, want_cid: bool = False):
    """O3: (count u64[K], sum f64[K,16], chk u64, cid int32[n] or None)."""
    x = np.ascontiguousarray(x, np.float32).reshape(-1, 16)
    mu = np.ascontiguousarray(mu, np.float32).reshape(-1, 16)
    K = mu.shape[0]
    count = np.empty(K, np.uint64); s = np.empty((K, 16), np.float64); chk = np.zeros(1, np.uint64)
    cid = np.empty(len(x), np.int32) if want_cid else None
    lib().oracle_kmeans(_p(x) if len(x) else None, len(x), _p(mu), K, first, _p(count), _p(s), _p(chk),
                        _p(cid) if want_cid and len(x) else None)
    return count, s, int(chk[0]), cid


def partition(kv, B: int = 1024):
    """O4: (boff u64[B+1], out u64[n,2]) stable by (bucket, index)."""
    kv = np.ascontiguousarray(kv, np.uint64).reshape(-1, 2)
    boff = np.empty(B + 1, np.uint64)
    out = np.empty_like(kv)
    rc = lib().oracle_partition(_p(kv) if len(kv) else None, len(kv), B, _p(boff), _p(out) if len(kv) else None)
    if rc:
        raise ValueError("B must be a power of two <= 65536")
    return boff, out


def groupby(recs, n: int, stride: int = 16, G: int = 4096):
    """O5: (count u64[G], qty u64[G], amount f64[G])."""
    r = _u8(recs)
    count = np.empty(G, np.uint64); qty = np.empty(G, np.uint64); amt = np.empty(G, np.float64)
    rc = lib().oracle_groupby(_p(r) if len(r) else None, n, stride, G, _p(count), _p(qty), _p(amt))
    if rc:
        raise ValueError("key >= G")
    return count, qty, amt


def kmer(recs, n: int, k: int = 31, rec_size: int = 256, seq_off: int = 16, seq_len: int = 96):
    """O6: (kmers u64 ascending, counts u64)."""
    r = _u8(recs)
    cap = 1 << 16
    while True:
        km = np.empty(cap, np.uint64); ct = np.empty(cap, np.uint64)
        V = lib().oracle_kmer(_p(r) if len(r) else None, n, rec_size, seq_off, seq_len, k, _p(km), _p(ct), cap)
        if V >= 0:
            return km[:V].copy(), ct[:V].copy()
        cap = -V


def _ext(extents):
    if not extents:
        return 0, None, None
    eo = np.array([e[0] for e in extents], np.uint32)
    el = np.array([e[1] for e in extents], np.uint32)
    return len(extents), eo, el


def plan_chunks(off, n: int, nbytes: int, rec_size: int, extents, budget: int) -> np.ndarray:
    """Greedy chunk bounds [0, ..., n] (whole records). Raises OverflowError on BK_E_RANGE."""
    ne, eo, el = _ext(extents)
    cap = n + 2
    bounds = np.empty(cap, np.uint64)
    offp = _p(np.ascontiguousarray(off, np.uint64)) if off is not None and len(off) else None
    C_ = lib().oracle_plan_chunks(offp, n, nbytes, rec_size, ne, _p(eo), _p(el), budget, _p(bounds), cap)
    if C_ == -1:
        raise OverflowError("record exceeds chunk budget")
    assert C_ >= 0
    return bounds[: C_ + 1].copy()


def layout(buf, off, n: int, nbytes: int, rec_size: int, extents, lo: int, hi: int, L: int, with_stage: bool = True):
    """O-L: (stage bytes, lane_first, lane_nrec, lane_bytes) for chunk [lo, hi) with L lanes."""
    ne, eo, el = _ext(extents)
    b = _u8(buf)
    offa = np.ascontiguousarray(off, np.uint64) if off is not None else None
    lf = np.empty(L, np.uint64); ln = np.empty(L, np.uint64); lb = np.empty(L, np.uint64)
    args = (_p(b) if len(b) else None, _p(offa) if offa is not None and len(offa) else None, n, nbytes, rec_size,
            ne, _p(eo), _p(el), lo, hi, L, _p(lf), _p(ln), _p(lb))
    size = lib().oracle_layout(*args, None, 0)
    if size < 0:
        raise ValueError("bad layout arguments")
    stage = None
    if with_stage:
        stage = np.empty(max(size, 1), np.uint8)
        size2 = lib().oracle_layout(*args, _p(stage), size)
        assert size2 == size
        stage = stage[:size]
    return stage, lf, ln, lb


def pattern_online(addrs, T: int = 8, pmax: int = 4):
    """O-P online: detect on the first T addresses, verify the rest; (base, strides) or None."""
    a = np.ascontiguousarray(addrs, np.uint64)
    st = np.empty(max(pmax, 1), np.int64)
    p = lib().oracle_pattern_online(_p(a) if len(a) else None, len(a), T, pmax, _p(st))
    if p == 0:
        return None
    return int(a[0]), [int(v) for v in st[:p]]


def pattern(addrs, pmax: int = 4):
    """O-P: (base, strides) or None."""
    a = np.ascontiguousarray(addrs, np.uint64)
    st = np.empty(max(pmax, 1), np.int64)
    p = lib().oracle_pattern(_p(a), len(a), pmax, _p(st))
    if p == 0:
        return None
    return int(a[0]), [int(v) for v in st[:p]]
