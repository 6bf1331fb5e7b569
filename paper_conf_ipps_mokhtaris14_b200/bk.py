"""Thin ctypes binding of libbk (include/bk.h): argument marshalling only.

Every step of the streaming path runs inside libbk.so (sm_100a kernels + C++ runtime). There
is no CPU fallback: if the library is missing or no GPU is present the calls raise.
Names follow the C ABI: bk_create / bk_register_segments / bk_run / bk_destroy.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libbk.so")

BK_OK, BK_E_INVAL, BK_E_NOMEM, BK_E_CUDA, BK_E_STATE, BK_E_RANGE, BK_E_CAPACITY, BK_E_UNSUPPORTED = 0, -1, -2, -3, -4, -5, -6, -7
BK_K_WORDCOUNT, BK_K_GREP, BK_K_KMEANS, BK_K_PARTITION, BK_K_GROUPBY, BK_K_LAYOUT_DUMP = 1, 2, 3, 4, 5, 100
BK_GATHER_AUTO, BK_GATHER_ZC, BK_GATHER_CPU, BK_GATHER_DENSE, BK_GATHER_HYBRID, BK_GATHER_FUSED, BK_GATHER_ADDR = (
    0, 1, 2, 3, 4, 5, 6)
BK_FLAG_PROFILE = 1
BK_FLAG_BASELINE_DBUF = 2
BK_FLAG_BASELINE_SBUF = 4
BK_FLAG_NO_GRAPH = 8
BK_FLAG_TEST_DELAYS = 16
BK_FLAG_KEEP_OUTPUTS_PINNED = 32
BK_FLAG_NO_PATTERNS = 64
BK_FLAG_TRACE = 128
GATHER_NAMES = {"auto": BK_GATHER_AUTO, "zc": BK_GATHER_ZC, "cpu": BK_GATHER_CPU, "dense": BK_GATHER_DENSE, "hybrid": BK_GATHER_HYBRID,
                "fused": BK_GATHER_FUSED, "addr": BK_GATHER_ADDR}

u32, i32, u64, P = C.c_uint32, C.c_int32, C.c_uint64, C.c_void_p


class bk_config(C.Structure):
    _fields_ = [("struct_size", u32), ("device", i32), ("window_bytes", u64), ("n_slots", u32),
                ("gather_mode", u32), ("chunk_bytes", u64), ("lanes", u32), ("host_threads", u32),
                ("record_size", u64), ("flags", u32), ("lane_bytes", u32),
                ("zc_share_pm", u32), ("addr_elem_bytes", u32)]


class bk_out_header(C.Structure):
    _fields_ = [("struct_size", u32), ("kernel_id", i32)]


class bk_out_wordcount(C.Structure):
    _fields_ = [("h", bk_out_header), ("table_slots", u64), ("cap", u64), ("word_off", P), ("word_len", P),
                ("word_count", P), ("n_words", u64), ("total_words", u64), ("word_h1", P), ("word_h2", P)]


class bk_out_grep(C.Structure):
    _fields_ = [("h", bk_out_header), ("pattern", P), ("pattern_len", u32), ("_pad", u32), ("first_index", u64),
                ("cap", u64), ("idx", P), ("n_match", u64)]


class bk_out_kmeans(C.Structure):
    _fields_ = [("h", bk_out_header), ("centroids", P), ("K", u32), ("_pad", u32), ("first_index", u64),
                ("count", P), ("sum", P), ("chk", u64), ("cid", P)]


class bk_out_partition(C.Structure):
    _fields_ = [("h", bk_out_header), ("n_buckets", u32), ("_pad", u32), ("out_records", P), ("chunk_counts", P),
                ("chunk_cap", u64), ("n_chunks", u64), ("bucket_count", P)]


class bk_out_groupby(C.Structure):
    _fields_ = [("h", bk_out_header), ("G", u32), ("_pad", u32), ("count", P), ("qty", P), ("amount", P)]


class bk_out_layout(C.Structure):
    _fields_ = [("h", bk_out_header), ("n_ext", u32), ("ext_off", u32 * 8), ("ext_len", u32 * 8), ("chunk", u64),
                ("stage", P), ("stage_cap", u64), ("lane_first", P), ("lane_nrec", P), ("lane_bytes", P),
                ("lane_cap", u64), ("stage_size", u64), ("lanes", u32), ("_pad", u32), ("chunk_lo", u64),
                ("chunk_hi", u64), ("n_chunks", u64)]


class bk_stats(C.Structure):
    _fields_ = [("struct_size", u32), ("gather_mode", u32), ("n_chunks", u64), ("chunk_budget", u64), ("lanes", u32),
                ("n_slots", u32), ("slot_bytes", u64), ("bytes_accessed", u64), ("bytes_h2d", u64),
                ("bytes_meta", u64), ("bytes_padding", u64), ("bytes_d2h", u64), ("kernel_launches", u64),
                ("ms_run", C.c_double), ("ms_register", C.c_double), ("ms_device", C.c_double),
                ("ms_h2d", C.c_double), ("ms_addrgen", C.c_double), ("ms_gather", C.c_double),
                ("ms_compute", C.c_double), ("n_gather", u64), ("n_chunks_cpu", u64), ("ms_cpu_gather", C.c_double),
                ("ms_xfer_busy", C.c_double), ("ms_compute_busy", C.c_double), ("ms_overlap", C.c_double),
                ("ms_zc", C.c_double), ("n_zc", u64), ("ms_relayout", C.c_double), ("n_relayout", u64),
                ("n_chunks_zc", u64), ("bytes_zc", u64), ("records_zc", u64), ("ms_d2h", C.c_double), ("n_d2h", u64),
                ("n_units", u64), ("unit_bytes", u32), ("fused_grid", u32), ("fused_loaders", u32),
                ("fused_ring_slots", u32), ("fused_wait_frac", C.c_double), ("fused_compute_frac", C.c_double),
                ("fused_loader_wait_frac", C.c_double), ("bytes_addr", u64), ("n_addr_lanes", u64),
                ("n_pattern_lanes", u64), ("n_addresses", u64), ("n_explicit_addr", u64), ("addr_elem_bytes", u32),
                ("_pad_addr", u32), ("ms_addr_wait", C.c_double), ("ms_trace_span", C.c_double),
                ("n_trace_records", u64), ("graph_issue", u32), ("_pad_graph", u32)]


class bk_out_pattern(C.Structure):
    _fields_ = [("h", bk_out_header), ("n_ext", u32), ("ext_off", u32 * 8), ("ext_len", u32 * 8), ("elem_bytes", u32),
                ("T", u32), ("pmax", u32), ("_pad", u32), ("chunk", u64), ("lane_p", P), ("lane_strides", P),
                ("lane_base", P), ("lane_count", P), ("lane_cap", u64), ("lanes", u32), ("_pad2", u32),
                ("n_lanes", u64), ("n_pattern_lanes", u64), ("n_addresses", u64), ("n_explicit_addresses", u64),
                ("address_bytes", u64), ("pattern_bytes", u64)]


class bk_out_kmer(C.Structure):
    _fields_ = [("h", bk_out_header), ("k", u32), ("seq_off", u32), ("seq_len", u32), ("_pad", u32),
                ("table_slots", u64), ("cap", u64), ("kmer", P), ("count", P), ("n_kmers", u64), ("total", u64)]


class bk_access(C.Structure):
    _fields_ = [("struct_size", u32), ("n_ext", u32), ("ext_off", u32 * 8), ("ext_len", u32 * 8), ("lane_bytes", u32),
                ("_reserved", u32)]


class bk_lane(C.Structure):
    _fields_ = [("first", u64), ("nrec", u32), ("nbytes", u32)]


class bk_chunk_view(C.Structure):
    _fields_ = [("struct_size", u32), ("lanes", u32), ("chunk_index", u64), ("n_chunks", u64),
                ("first_record", u64), ("n_records", u64), ("stage", P), ("lane_desc", P), ("tile_base", P),
                ("offsets", P), ("end_offset", u64)]


class bk_addr_view(C.Structure):
    _fields_ = [("struct_size", u32), ("lanes", u32), ("chunk_index", u64), ("n_chunks", u64),
                ("first_record", u64), ("n_records", u64), ("lane_desc", P), ("offsets", P), ("end_offset", u64),
                ("addr", P), ("addr_base", P), ("addr_count", P), ("elem_bytes", u32), ("_pad", u32)]


# int (*bk_chunk_fn)(const bk_chunk_view* view, void* stream, void* user)
bk_chunk_fn = C.CFUNCTYPE(C.c_int, C.POINTER(bk_chunk_view), P, P)
bk_addr_fn = C.CFUNCTYPE(C.c_int, C.POINTER(bk_addr_view), P, P)

BK_K_PATTERN_STATS = 101
BK_K_KMER = 6
ABI_STRUCTS = [bk_config, bk_out_wordcount, bk_out_grep, bk_out_kmeans, bk_out_partition, bk_out_groupby,
               bk_out_layout, bk_stats, bk_out_pattern, bk_out_kmer, bk_access, bk_chunk_view, bk_addr_view]
EXPORTS = ["bk_create", "bk_register_segments", "bk_run", "bk_run_user", "bk_destroy", "bk_strerror",
           "bk_last_error", "bk_get_stats", "bk_abi_sizes", "bk_partition_materialize", "bk_unpin_outputs",
           "bk_merge_counts", "bk_run_user_addr"]

_lib = None


class BkError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        detail = lib().bk_last_error().decode(errors="replace")
        super().__init__(f"{where}: {lib().bk_strerror(status).decode()} ({status}): {detail}")


def lib() -> C.CDLL:
    """Load libbk.so. Fails loudly when it is missing: there is no fallback path."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} not built; run `make` or __graft_entry__.build()")
        l = C.CDLL(LIB_PATH)
        l.bk_create.argtypes = [C.POINTER(bk_config), C.POINTER(P)]
        l.bk_register_segments.argtypes = [P, P, u64, P, u64]
        l.bk_run.argtypes = [P, C.c_int, P, P]
        l.bk_destroy.argtypes = [P]
        l.bk_strerror.argtypes = [C.c_int]
        l.bk_strerror.restype = C.c_char_p
        l.bk_last_error.argtypes = []
        l.bk_last_error.restype = C.c_char_p
        l.bk_get_stats.argtypes = [P, C.POINTER(bk_stats)]
        l.bk_abi_sizes.argtypes = [C.POINTER(u32), C.c_int]
        l.bk_run_user.argtypes = [P, C.POINTER(bk_access), P, P, P]
        l.bk_partition_materialize.argtypes = [P, P, u64, u32, P, P, u32]
        l.bk_unpin_outputs.argtypes = [P]
        l.bk_merge_counts.argtypes = [P, P, u32, u64, P, u32, u32, u32, P, u64, C.POINTER(u64), P]
        l.bk_run_user_addr.argtypes = [P, C.POINTER(bk_access), P, P, P, P, P]
        for name in ("bk_create", "bk_register_segments", "bk_run", "bk_run_user", "bk_destroy", "bk_get_stats",
                     "bk_abi_sizes", "bk_partition_materialize", "bk_unpin_outputs", "bk_merge_counts",
                     "bk_run_user_addr"):
            getattr(l, name).restype = C.c_int
        _lib = l
    return _lib


def check(status: int, where: str) -> None:
    if status != BK_OK:
        raise BkError(status, where)


def abi_sizes() -> list[int]:
    a = (u32 * len(ABI_STRUCTS))()
    lib().bk_abi_sizes(a, len(ABI_STRUCTS))
    return list(a)


def _ptr(a) -> int | None:
    """Address of a numpy array, a torch tensor (host or device memory: the aggregating kernels'
    result arrays may live on the context's GPU, bk.h) or a raw integer address."""
    if a is None:
        return None
    if isinstance(a, np.ndarray):
        assert a.flags["C_CONTIGUOUS"]
        return a.ctypes.data
    if hasattr(a, "data_ptr"):
        assert a.is_contiguous()
        return a.data_ptr()
    return int(a)


def bk_create(device: int = 0, window_bytes: int = 0, n_slots: int = 0, gather_mode: int | str = 0,
              chunk_bytes: int = 0, lanes: int = 0, record_size: int = 0, host_threads: int = 0,
              profile: bool = False, baseline_dbuf: bool = False, lane_bytes: int = 0,
              zc_share_pm: int = 0, baseline_sbuf: bool = False, no_graph: bool = False,
              test_delays: bool = False, keep_outputs_pinned: bool = False, no_patterns: bool = False,
              addr_elem_bytes: int = 0, trace: bool = False) -> int:
    if isinstance(gather_mode, str):
        gather_mode = GATHER_NAMES[gather_mode]
    cfg = bk_config(C.sizeof(bk_config), device, window_bytes, n_slots, gather_mode, chunk_bytes, lanes,
                    host_threads, record_size,
                    (BK_FLAG_PROFILE if profile else 0) | (BK_FLAG_BASELINE_DBUF if baseline_dbuf else 0) |
                    (BK_FLAG_BASELINE_SBUF if baseline_sbuf else 0) | (BK_FLAG_NO_GRAPH if no_graph else 0) |
                    (BK_FLAG_TEST_DELAYS if test_delays else 0) |
                    (BK_FLAG_KEEP_OUTPUTS_PINNED if keep_outputs_pinned else 0) |
                    (BK_FLAG_NO_PATTERNS if no_patterns else 0) | (BK_FLAG_TRACE if trace else 0),
                    lane_bytes,
                    zc_share_pm, addr_elem_bytes)
    ctx = P()
    check(lib().bk_create(C.byref(cfg), C.byref(ctx)), "bk_create")
    return ctx.value


def bk_register_segments(ctx: int, data, offsets=None, nbytes: int | None = None, n_records: int | None = None) -> None:
    """data: uint8 ndarray (or raw host address with nbytes); offsets: uint64 ndarray or None."""
    nb = nbytes if nbytes is not None else int(data.nbytes)
    if offsets is not None:
        assert offsets.dtype == np.uint64
        n = len(offsets) if n_records is None else n_records
    else:
        n = n_records if n_records is not None else 0
    check(lib().bk_register_segments(ctx, _ptr(data), nb, _ptr(offsets) if offsets is not None and len(offsets) else None, n),
          "bk_register_segments")


def bk_run(ctx: int, kernel_id: int, stream, out) -> None:
    check(lib().bk_run(ctx, kernel_id, stream, C.byref(out)), "bk_run")


def partition_materialize(out: np.ndarray, chunk_counts: np.ndarray, bucket_start: np.ndarray | None = None,
                          dst: np.ndarray | None = None, threads: int = 0) -> np.ndarray:
    """bk_partition_materialize: chunk-major runs (Context.partition) -> bucket-major stable order.
    dst defaults to a new n x 2 u64 array (bucket_start None: local offsets)."""
    cc = np.ascontiguousarray(chunk_counts, np.uint64)
    C, B = cc.shape
    if dst is None:
        dst = np.empty((int(cc.sum()), 2), np.uint64)
    bs = None if bucket_start is None else np.ascontiguousarray(bucket_start, np.uint64)
    check(lib().bk_partition_materialize(_ptr(out) if C else None, _ptr(cc) if C else None, C, B,
                                         _ptr(bs) if bs is not None else None, _ptr(dst) if C else None, threads),
          "bk_partition_materialize")
    return dst


def bk_destroy(ctx: int) -> None:
    check(lib().bk_destroy(ctx), "bk_destroy")


def bk_get_stats(ctx: int) -> dict:
    s = bk_stats()
    s.struct_size = C.sizeof(bk_stats)
    check(lib().bk_get_stats(ctx, C.byref(s)), "bk_get_stats")
    return {k: getattr(s, k) for k, _ in bk_stats._fields_ if k != "struct_size"}


def _hdr(cls, kid):
    o = cls()
    o.h.struct_size = C.sizeof(cls)
    o.h.kernel_id = kid
    return o


class Context:
    """Owning wrapper: one context per GPU; marshals the per-kernel in/out structs."""

    def __init__(self, **cfg):
        self.ctx = bk_create(**cfg)
        self._keep = []

    def close(self):
        if self.ctx:
            bk_destroy(self.ctx)
            self.ctx = None

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def register(self, data, offsets=None, n_records=None, nbytes=None):
        self._keep = [data, offsets]
        self.n = len(offsets) if offsets is not None else (n_records or 0)
        bk_register_segments(self.ctx, data, offsets, nbytes=nbytes, n_records=n_records)

    def stats(self) -> dict:
        return bk_get_stats(self.ctx)

    def unpin_outputs(self):
        """bk_unpin_outputs: release output arrays kept pinned (keep_outputs_pinned=True)."""
        check(lib().bk_unpin_outputs(self.ctx), "bk_unpin_outputs")

    def wordcount(self, cap: int = 1 << 20, table_slots: int = 0, stream=None, out=None):
        """(word_off u64, word_len u32, word_count u64) of every distinct word; `out`: optional
        preallocated (off, len, count) or (off, len, count, h1, h2) arrays of equal length (the cap),
        numpy or torch (host or device), reused across calls; with h1/h2 the word identities (the
        multi-GPU merge key) are returned too."""
        o = _hdr(bk_out_wordcount, BK_K_WORDCOUNT)
        if out is not None:
            assert len(out) in (3, 5) and len({len(a) for a in out}) == 1
            cap = len(out[0])
        else:
            out = (np.empty(cap, np.uint64), np.empty(cap, np.uint32), np.empty(cap, np.uint64))
        o.table_slots, o.cap = table_slots, cap
        o.word_off, o.word_len, o.word_count = _ptr(out[0]), _ptr(out[1]), _ptr(out[2])
        if len(out) == 5:
            o.word_h1, o.word_h2 = _ptr(out[3]), _ptr(out[4])
        bk_run(self.ctx, BK_K_WORDCOUNT, stream, o)
        self.total_words = int(o.total_words)
        n = o.n_words
        return tuple(a[:n] for a in out)

    def grep(self, pattern: bytes = b"bigk", first_index: int = 0, cap: int | None = None, stream=None, out=None):
        o = _hdr(bk_out_grep, BK_K_GREP)
        pat = np.frombuffer(pattern, np.uint8) if pattern else np.zeros(1, np.uint8)
        idx = out if out is not None else np.empty(max(cap or 1 << 20, 1), np.uint64)
        o.pattern, o.pattern_len, o.first_index, o.cap, o.idx = _ptr(pat), len(pattern), first_index, len(idx), _ptr(idx)
        bk_run(self.ctx, BK_K_GREP, stream, o)
        return idx[: o.n_match]

    def groupby(self, G: int = 4096, stream=None, out=None):
        """(count u64[G], qty u64[G], amount f64[G]); `out`: optional (count, qty, amount) arrays,
        numpy or torch (host or device memory of this context's GPU)."""
        o = _hdr(bk_out_groupby, BK_K_GROUPBY)
        if out is None:
            out = (np.empty(G, np.uint64), np.empty(G, np.uint64), np.empty(G, np.float64))
        assert all(len(a) >= G for a in out)
        o.G, o.count, o.qty, o.amount = G, _ptr(out[0]), _ptr(out[1]), _ptr(out[2])
        bk_run(self.ctx, BK_K_GROUPBY, stream, o)
        return out

    def kmeans(self, mu: np.ndarray, first_index: int = 0, stream=None, cid=None, out=None):
        """(count u64[K], sum f64[K,16], chk); cid: optional int32[n] (host) written back per record;
        out: optional (count[K], sum[K*16 or K,16]) arrays, numpy or torch (host or device)."""
        mu = np.ascontiguousarray(mu, np.float32).reshape(-1, 16)
        K = mu.shape[0]
        o = _hdr(bk_out_kmeans, BK_K_KMEANS)
        if out is None:
            out = (np.empty(K, np.uint64), np.empty((K, 16), np.float64))
        cnt, s = out
        if cid is not None:
            assert cid.dtype == np.int32 and len(cid) >= self.n
        o.centroids, o.K, o.first_index, o.count, o.sum = _ptr(mu), K, first_index, _ptr(cnt), _ptr(s)
        o.cid = _ptr(cid) if cid is not None and self.n else None
        bk_run(self.ctx, BK_K_KMEANS, stream, o)
        return cnt, s, int(o.chk)

    def merge_counts(self, rows, seg_rows, seg_stride: int, row_u64: int, key_u64: int, count_col: int, out,
                     stream=None) -> int:
        """bk_merge_counts over DEVICE arrays (torch tensors on this context's GPU): `rows` holds
        len(seg_rows) segments of seg_stride rows; merged rows go to `out` (cap = its rows).
        Returns the number of distinct keys."""
        segs = np.ascontiguousarray(seg_rows, np.uint64)
        cap = out.numel() // row_u64 if hasattr(out, "numel") else len(out) // row_u64
        n = u64(0)
        check(lib().bk_merge_counts(self.ctx, _ptr(rows), len(segs), seg_stride, _ptr(segs), row_u64, key_u64,
                                    count_col, _ptr(out), cap, C.byref(n), stream), "bk_merge_counts")
        return int(n.value)

    def partition(self, n_buckets: int = 1024, out=None, chunk_cap: int = 1 << 16, stream=None):
        """Returns (out u64[n,2] chunk-major bucket-sorted runs, chunk_counts u64[C,B], bucket_count u64[B])."""
        o = _hdr(bk_out_partition, BK_K_PARTITION)
        out = out if out is not None else np.empty((self.n, 2), np.uint64)
        cc = np.empty(chunk_cap * n_buckets, np.uint64)
        bc = np.empty(n_buckets, np.uint64)
        o.n_buckets, o.out_records, o.chunk_counts, o.chunk_cap, o.bucket_count = (
            n_buckets, _ptr(out) if self.n else None, _ptr(cc), chunk_cap, _ptr(bc))
        bk_run(self.ctx, BK_K_PARTITION, stream, o)
        C = o.n_chunks
        return out, cc[: C * n_buckets].reshape(C, n_buckets), bc

    def kmer(self, k: int = 31, seq_off: int = 16, seq_len: int = 96, table_slots: int = 0, cap: int = 1 << 22,
             stream=None, out=None):
        """f4: (kmers u64, counts u64) unordered, and the total number of k-mer occurrences.
        out: optional preallocated (kmers, counts) arrays of equal length (the capacity)."""
        o = _hdr(bk_out_kmer, BK_K_KMER)
        if out is not None:
            km, ct = out
            cap = min(len(km), len(ct))
        else:
            km = np.empty(cap, np.uint64); ct = np.empty(cap, np.uint64)
        o.k, o.seq_off, o.seq_len, o.table_slots, o.cap, o.kmer, o.count = k, seq_off, seq_len, table_slots, cap, \
            _ptr(km), _ptr(ct)
        bk_run(self.ctx, BK_K_KMER, stream, o)
        return km[: o.n_kmers], ct[: o.n_kmers], int(o.total)

    def pattern_stats(self, extents=None, elem_bytes: int = 1, T: int = 8, pmax: int = 4, chunk: int | None = None,
                      lane_cap: int = 1 << 20, stream=None):
        """Stage 1 in address mode + online pattern recognition over every lane.
        Returns the totals dict and, for `chunk`, per-lane (p, strides[4], base, count)."""
        o = _hdr(bk_out_pattern, BK_K_PATTERN_STATS)
        extents = extents or []
        o.n_ext = len(extents)
        for i, (eo, el) in enumerate(extents):
            o.ext_off[i], o.ext_len[i] = eo, el
        o.elem_bytes, o.T, o.pmax = elem_bytes, T, pmax
        p_ = np.empty(lane_cap, np.int32); st = np.empty((lane_cap, 4), np.int64)
        base = np.empty(lane_cap, np.uint64); cnt = np.empty(lane_cap, np.uint64)
        o.chunk = chunk if chunk is not None else (1 << 64) - 1
        o.lane_p, o.lane_strides, o.lane_base, o.lane_count, o.lane_cap = _ptr(p_), _ptr(st), _ptr(base), _ptr(cnt), lane_cap
        bk_run(self.ctx, BK_K_PATTERN_STATS, stream, o)
        tot = {k: getattr(o, k) for k in ("n_lanes", "n_pattern_lanes", "n_addresses", "n_explicit_addresses",
                                          "address_bytes", "pattern_bytes", "lanes")}
        L = o.lanes
        lanes = (p_[:L].copy(), st[:L].copy(), base[:L].copy(), cnt[:L].copy()) if chunk is not None else None
        return tot, lanes

    def run_user(self, fn, user=None, extents=None, lane_bytes: int = 0, stream=None):
        """bk_run_user: stages 1-3 under `extents` ([(offset, length), ...]; None = whole records),
        then fn(view*, stream, user) per chunk enqueues the caller's own stage-4 kernel. `fn` is a
        native bk_chunk_fn (e.g. a symbol of the caller's CUDA library) or a bk_chunk_fn wrapper;
        `user` an opaque pointer (int address or ctypes object) handed back to it."""
        a = bk_access()
        a.struct_size = C.sizeof(bk_access)
        extents = extents or []
        a.n_ext = len(extents)
        for i, (eo, el) in enumerate(extents):
            a.ext_off[i], a.ext_len[i] = eo, el
        a.lane_bytes = lane_bytes
        fp = C.cast(fn, P)
        up = user if (user is None or isinstance(user, int)) else C.cast(C.pointer(user), P)
        check(lib().bk_run_user(self.ctx, C.byref(a), fp, up, stream), "bk_run_user")

    def run_user_addr(self, gen, fn, gen_user=None, user=None, bound=None, lane_bytes: int = 0, stream=None):
        """bk_run_user_addr: `gen` (a native bk_addr_fn) writes every lane's element addresses per chunk
        (stage 1), libbk recognises patterns, ships addresses, assembles and DMAs (stages 2-3), then
        `fn` (a native bk_chunk_fn) enqueues stage 4. `bound`: [(offset, length), ...] per record
        bounding the lanes' capacities (None = whole records)."""
        a = bk_access()
        a.struct_size = C.sizeof(bk_access)
        bound = bound or []
        a.n_ext = len(bound)
        for i, (eo, el) in enumerate(bound):
            a.ext_off[i], a.ext_len[i] = eo, el
        a.lane_bytes = lane_bytes
        gu = gen_user if (gen_user is None or isinstance(gen_user, int)) else C.cast(C.pointer(gen_user), P)
        up = user if (user is None or isinstance(user, int)) else C.cast(C.pointer(user), P)
        check(lib().bk_run_user_addr(self.ctx, C.byref(a), C.cast(gen, P), gu, C.cast(fn, P), up, stream),
              "bk_run_user_addr")

    def layout_dump(self, chunk: int, extents=None, stage_cap: int = 1 << 26, lane_cap: int = 1 << 20, stream=None):
        o = _hdr(bk_out_layout, BK_K_LAYOUT_DUMP)
        extents = extents or []
        o.n_ext = len(extents)
        for i, (eo, el) in enumerate(extents):
            o.ext_off[i], o.ext_len[i] = eo, el
        stage = np.empty(stage_cap, np.uint8)
        lf = np.empty(lane_cap, np.uint64); ln = np.empty(lane_cap, np.uint64); lb = np.empty(lane_cap, np.uint64)
        o.chunk, o.stage, o.stage_cap = chunk, _ptr(stage), stage_cap
        o.lane_first, o.lane_nrec, o.lane_bytes, o.lane_cap = _ptr(lf), _ptr(ln), _ptr(lb), lane_cap
        bk_run(self.ctx, BK_K_LAYOUT_DUMP, stream, o)
        L = o.lanes
        return dict(stage=stage[: o.stage_size].copy(), lane_first=lf[:L].copy(), lane_nrec=ln[:L].copy(),
                    lane_bytes=lb[:L].copy(), lanes=L, lo=o.chunk_lo, hi=o.chunk_hi, n_chunks=o.n_chunks)
