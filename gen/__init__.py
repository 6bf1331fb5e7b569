"""Seeded synthetic input generators (ctypes over gen/libbkgen.so).

Input generation only: both the CUDA path's tests/bench and the oracle
consume these bytes; nothing here is part of either computation. Counter-based RNG, so any
record range (a GPU shard) regenerates independently and identically.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libbkgen.so")
_SRC = os.path.join(_HERE, "gen.c")

SEED_WC = 0xB16C0001
SEED_GREP = 0xB16C0002
SEED_KMEANS = 0xB16C0003
SEED_KV = 0xB16C0004
SEED_GROUPBY = 0xB16C0005
SEED_DNA = 0xB16C0006

_lib = None


def build() -> str:
    if not os.path.exists(_SO) or os.path.getmtime(_SO) < max(os.path.getmtime(_SRC), os.path.getmtime(_SRC[:-1] + "h")):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-Wall", _SRC, "-o", _SO, "-lm"])
    return _SO


def lib():
    global _lib
    if _lib is None:
        l = C.CDLL(build())
        u64, p = C.c_uint64, C.c_void_p
        l.gen_R.restype = u64
        l.gen_R.argtypes = [u64, u64, u64]
        l.gen_text.restype = C.c_int
        l.gen_text.argtypes = [u64, u64, p, p, u64, p, p]
        l.gen_grep_sizes.restype = u64
        l.gen_grep_sizes.argtypes = [u64, u64, u64, p]
        l.gen_grep_count_for_bytes.restype = u64
        l.gen_grep_count_for_bytes.argtypes = [u64, u64, u64]
        l.gen_grep_fill.restype = None
        l.gen_grep_fill.argtypes = [u64, u64, u64, p, p, C.c_int]
        l.gen_points.restype = None
        l.gen_points.argtypes = [u64, u64, u64, p, C.c_int]
        l.gen_kv.restype = None
        l.gen_kv.argtypes = [u64, u64, u64, p, C.c_int]
        l.gen_groupby.restype = None
        l.gen_groupby.argtypes = [u64, u64, u64, C.c_uint32, C.c_uint32, C.c_int, p, C.c_int]
        l.gen_dna.restype = None
        l.gen_dna.argtypes = [u64, u64, u64, u64, C.c_uint32, C.c_uint32, p, C.c_int]
        l.gen_alloc.restype = p
        l.gen_alloc.argtypes = [u64, C.c_int, C.POINTER(p), C.POINTER(u64)]
        l.gen_free.restype = None
        l.gen_free.argtypes = [p, u64]
        _lib = l
    return _lib


def _threads(threads):
    return threads if threads else (len(os.sched_getaffinity(0)) or 1)


def _ptr(a: np.ndarray) -> int:
    assert a.flags["C_CONTIGUOUS"]
    return a.ctypes.data


def dna(seed: int = SEED_DNA, first: int = 0, n: int = 1 << 16, genome_len: int = 1 << 20, err_pm: int = 1,
        n_pm: int = 2, out: np.ndarray | None = None, threads: int = 0):
    """f4: n x 256-B read records (96-base sequence at +16) sampled from a seeded genome."""
    buf = out if out is not None else np.empty(n * 256, np.uint8)
    lib().gen_dna(seed, first, n, genome_len, err_pm, n_pm, _ptr(buf), _threads(threads))
    return buf


class _Mapping:
    """Owner of a gen_alloc mapping; numpy views keep it (their ultimate .base) alive."""

    def __init__(self, p: int, n: int, base: int, ln: int):
        self.__array_interface__ = {"data": (p, False), "shape": (n,), "typestr": "|u1", "version": 3}
        self._region = (base, ln)

    def __del__(self):
        lib().gen_free(*self._region)


def alloc(nbytes: int, huge: bool = True) -> np.ndarray:
    """uint8 array of nbytes in a 2 MiB-aligned mapping (transparent huge pages when huge)."""
    base, ln = C.c_void_p(), C.c_uint64()
    p = lib().gen_alloc(max(nbytes, 1), int(huge), C.byref(base), C.byref(ln))
    if not p:
        raise MemoryError(nbytes)
    return np.asarray(_Mapping(p, nbytes, base.value, ln.value))


def R(seed: int, stream: int, i: int) -> int:
    return lib().gen_R(seed, stream, i)


def text(seed: int = SEED_WC, cap_bytes: int = 64 << 20, cap_recs: int | None = None):
    """C1: Zipf word lines. Returns (buf uint8[nbytes], off uint64[n])."""
    cap_recs = cap_recs if cap_recs is not None else cap_bytes + 1
    buf = np.empty(cap_bytes, np.uint8)
    off = np.empty(min(cap_recs, cap_bytes + 1), np.uint64)
    nb, nr = C.c_uint64(), C.c_uint64()
    rc = lib().gen_text(seed, cap_bytes, _ptr(buf), _ptr(off), len(off), C.byref(nb), C.byref(nr))
    assert rc == 0
    return buf[: nb.value].copy(), off[: nr.value].copy()


def grep_count_for_bytes(seed: int, first: int, max_bytes: int) -> int:
    return lib().gen_grep_count_for_bytes(seed, first, max_bytes)


def grep_records(seed: int = SEED_GREP, first: int = 0, n: int | None = None, max_bytes: int | None = None,
                 out: np.ndarray | None = None, threads: int = 0):
    """C2: variable-length records (A16). Returns (buf uint8[nbytes], off uint64[n])."""
    if n is None:
        n = grep_count_for_bytes(seed, first, max_bytes)
    off = np.empty(n, np.uint64)
    nbytes = lib().gen_grep_sizes(seed, first, n, _ptr(off))
    buf = out[:nbytes] if out is not None else np.empty(nbytes, np.uint8)
    lib().gen_grep_fill(seed, first, n, _ptr(off), _ptr(buf), _threads(threads))
    return buf, off


def points(seed: int = SEED_KMEANS, first: int = 0, n: int = 1 << 20, out: np.ndarray | None = None, threads: int = 0):
    """C3: n x 16 fp32 points."""
    x = out if out is not None else np.empty((n, 16), np.float32)
    lib().gen_points(seed, first, n, _ptr(x), _threads(threads))
    return x


def kv(seed: int = SEED_KV, first: int = 0, n: int = 1 << 20, out: np.ndarray | None = None, threads: int = 0):
    """C4: n x {u64 key, u64 value=i}."""
    a = out if out is not None else np.empty((n, 2), np.uint64)
    lib().gen_kv(seed, first, n, _ptr(a), _threads(threads))
    return a


def groupby(seed: int = SEED_GROUPBY, first: int = 0, n: int = 1 << 20, G: int = 4096, stride: int = 16,
            zipf: bool = False, out: np.ndarray | None = None, threads: int = 0):
    """C5: n records {u32 key<G, u32 qty, f64 amount} at `stride` bytes (16 dense, 64 sparse)."""
    buf = out if out is not None else np.empty(n * stride, np.uint8)
    lib().gen_groupby(seed, first, n, G, stride, int(zipf), _ptr(buf), _threads(threads))
    return buf
