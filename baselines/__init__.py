"""The paper's multithreaded CPU variant (ii), bench-only (ctypes over
baselines/libbkmt.so, OpenMP on all host cores). Not the oracle, not part of libbk."""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libbkmt.so")
_SRC = os.path.join(_HERE, "cpu_mt.c")
_lib = None


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
            subprocess.check_call(["gcc", "-O3", "-march=x86-64-v3", "-ffp-contract=off", "-fopenmp", "-fPIC",
                                   "-shared", _SRC, "-o", _SO, "-lm"])
        l = C.CDLL(_SO)
        p, u64, u32 = C.c_void_p, C.c_uint64, C.c_uint32
        l.mt_threads.restype = C.c_int
        l.mt_set_threads.argtypes = [C.c_int]
        l.mt_grep.restype = C.c_int64
        l.mt_grep.argtypes = [p, u64, p, u64, p, u32, p, u64]
        l.mt_groupby.argtypes = [p, u64, u32, u32, p, p, p]
        l.mt_kmeans.argtypes = [p, u64, p, u32, p, p]
        l.mt_partition.argtypes = [p, u64, u32, p, p]
        l.mt_wordcount.restype = C.c_int64
        l.mt_wordcount.argtypes = [p, u64, p, u64, p, p, p, u64]
        l.mt_kmer.restype = C.c_int64
        l.mt_kmer.argtypes = [p, u64, u32, u32, u32, u32, u64, p, p, u64]
        l.mt_stream_copy.restype = C.c_double
        l.mt_stream_copy.argtypes = [p, p, u64, C.c_int]
        l.mt_stream_read.restype = C.c_double
        l.mt_stream_read.argtypes = [p, u64, C.c_int, p]
        _lib = l
    return _lib


def threads() -> int:
    return lib().mt_threads()


def set_threads(n: int) -> None:
    """OpenMP thread count of the baseline (torchrun sets OMP_NUM_THREADS=1 for N > 1 ranks)."""
    lib().mt_set_threads(int(n))


def grep(buf, off, pattern: bytes = b"bigk"):
    pat = np.frombuffer(pattern, np.uint8) if pattern else np.zeros(1, np.uint8)
    idx = np.empty(max(len(off), 1), np.uint64)
    m = lib().mt_grep(buf.ctypes.data, len(buf), off.ctypes.data, len(off), pat.ctypes.data, len(pattern),
                      idx.ctypes.data, len(idx))
    return idx[:m]


def groupby(buf, n, stride=16, G=4096):
    c = np.empty(G, np.uint64); q = np.empty(G, np.uint64); a = np.empty(G, np.float64)
    lib().mt_groupby(buf.ctypes.data, n, stride, G, c.ctypes.data, q.ctypes.data, a.ctypes.data)
    return c, q, a


def kmeans(x, mu):
    mu = np.ascontiguousarray(mu, np.float32)
    K = mu.shape[0]
    c = np.empty(K, np.uint64); s = np.empty((K, 16), np.float64)
    lib().mt_kmeans(x.ctypes.data, len(x), mu.ctypes.data, K, c.ctypes.data, s.ctypes.data)
    return c, s


def partition(kv, B=1024):
    """(boff u64[B+1], out u64[n,2]) stable bucket-major, like oracle.partition."""
    kv = np.ascontiguousarray(kv, np.uint64).reshape(-1, 2)
    out = np.empty_like(kv)
    boff = np.empty(B + 1, np.uint64)
    lib().mt_partition(kv.ctypes.data, len(kv), B, out.ctypes.data, boff.ctypes.data)
    return boff, out


def kmer(recs, n, k=31, rec_size=256, seq_off=16, seq_len=96, slots=None):
    """(kmers u64 ascending, counts u64), like oracle.kmer."""
    slots = slots or 1 << max(16, int(2 * n * (seq_len - k + 1)).bit_length())
    cap = 1 << 16
    while True:
        km = np.empty(cap, np.uint64); ct = np.empty(cap, np.uint64)
        V = lib().mt_kmer(recs.ctypes.data, n, rec_size, seq_off, seq_len, k, slots, km.ctypes.data, ct.ctypes.data,
                          cap)
        if V == -1:
            raise RuntimeError("k-mer table full")
        if V >= 0:
            o = np.argsort(km[:V])
            return km[:V][o], ct[:V][o]
        cap = -V


def wordcount(buf, off):
    """(word_off u64, word_len u32, count u64) of every distinct word, unordered (like the GPU's)."""
    cap = 1 << 17
    while True:
        wo = np.empty(cap, np.uint64); wl = np.empty(cap, np.uint32); wc = np.empty(cap, np.uint64)
        V = lib().mt_wordcount(buf.ctypes.data, len(buf), off.ctypes.data, len(off), wo.ctypes.data, wl.ctypes.data,
                               wc.ctypes.data, cap)
        if V >= 0:
            return wo[:V], wl[:V], wc[:V]
        cap = -V


def host_stream(gib: float = 2.0, reps: int = 3) -> dict:
    """Host DRAM bandwidth on all OpenMP threads (bench.py's host roofline): STREAM-style copy
    (bytes read + written per second) and read-only, over buffers far larger than the LLC."""
    n = int(gib * (1 << 30))
    a = np.ones(n, np.uint8)
    b = np.empty(n, np.uint8)
    b.fill(1)
    sink = np.zeros(1, np.uint64)
    cp = lib().mt_stream_copy(a.ctypes.data, b.ctypes.data, n, reps)
    rd = lib().mt_stream_read(a.ctypes.data, n, reps, sink.ctypes.data)
    return {"copy_gbs": cp / 1e9, "read_gbs": rd / 1e9, "threads": threads(), "gib": gib}
