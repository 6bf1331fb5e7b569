/* bk.h — C ABI of libbk, the B200-native BigKernel streaming path.
 *
 * What it implements (§III): a kernel over an arbitrarily large,
 * record-partitioned host data set ("segments") runs as a four-stage pipeline —
 *   (1) prefetch address generation on the GPU,
 *   (2) assembly of exactly the accessed bytes in thread-interleaved order,
 *   (3) transfer over the host link,
 *   (4) the compute kernel over the staged chunk,
 * with several buffer instances so the stages of consecutive chunks overlap.
 * The programmer registers the host array once and calls bk_run once; there are no
 * programmer-managed buffers, chunks or transfers.
 *
 * Plain C: no CUDA, PyTorch or C++ types in any signature. A CUDA stream is passed as an
 * opaque `void*` (a cudaStream_t / CUstream; NULL = legacy default stream). Every function
 * returns a bk_status (0 = OK, negative = error); no exception or CUDA error escapes.
 * bk_last_error() returns a thread-local detail string for the most recent failure.
 * A context is single-threaded: use one context per GPU (several per process are allowed).
 */
#ifndef BK_H
#define BK_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

#define BK_ABI_VERSION 2
#if defined(__GNUC__)
#define BK_API __attribute__((visibility("default")))
#else
#define BK_API
#endif

typedef enum {
  BK_OK = 0,
  BK_E_INVAL = -1,        /* bad argument, malformed offsets, key out of range */
  BK_E_NOMEM = -2,        /* device or pinned allocation failed / window too small */
  BK_E_CUDA = -3,         /* CUDA runtime/driver error (detail in bk_last_error) */
  BK_E_STATE = -4,        /* call out of order (run before register, ...) */
  BK_E_RANGE = -5,        /* one record's accessed bytes exceed the chunk budget (A18) */
  BK_E_CAPACITY = -6,     /* output or table too small; required size written back */
  BK_E_UNSUPPORTED = -7   /* kernel id / gather mode not supported by this build */
} bk_status;

/* Built-in compute kernels (north_star: kernels selected by kernel_id). */
typedef enum {
  BK_K_WORDCOUNT = 1,   /* C1: word -> count table        out: bk_out_wordcount */
  BK_K_GREP = 2,        /* C2: ordered indices of records whose key contains a pattern bk_out_grep */
  BK_K_KMEANS = 3,      /* C3: assignment + per-cluster partial sums      bk_out_kmeans */
  BK_K_PARTITION = 4,   /* C4: stable hash partition into B buckets                    bk_out_partition */
  BK_K_GROUPBY = 5,     /* C5: group-by count / sum                                    bk_out_groupby */
  BK_K_KMER = 6,        /* f4: k-mer counting over fixed-length DNA reads           bk_out_kmer */
  BK_K_LAYOUT_DUMP = 100, /* test only: copy one chunk's staged bytes + lane table back      bk_out_layout */
  BK_K_PATTERN_STATS = 101 /* stage 1 in address mode + online pattern recognition over
                              every lane's element-address stream; Table II accounting     bk_out_pattern */
} bk_kernel_id;

/* Stage-2/3 implementations. */
typedef enum {
  BK_GATHER_AUTO = 0,   /* HYBRID for sparse access, DENSE when every byte is accessed */
  BK_GATHER_ZC = 1,     /* GPU kernel reads the accessed bytes from pinned, mapped host memory
                           (16-B loads) and writes the interleaved tiles to HBM: stages 2+3 fused */
  BK_GATHER_CPU = 2,    /* a host thread pool packs exactly the accessed bytes into pinned staging in
                           the warp-tile layout (the paper's CPU assembly), then one DMA */
  BK_GATHER_DENSE = 3,  /* one contiguous DMA of the chunk's records (copy engine), then an
                           HBM->HBM re-layout kernel (fetch-all) */
  BK_GATHER_HYBRID = 4, /* chunks split between the GPU zero-copy gather and CPU assembly, running
                           concurrently and sharing the link (see zc_share_pm) */
  BK_GATHER_FUSED = 5,  /* BK_K_WORDCOUNT only (AUTO picks it there): the whole run is ONE persistent,
                           cooperative kernel (the paper's single launch): loader CTAs copy
                           each unit of whole records (offsets + bytes, zero-copy) into a ring in the
                           window and publish it with a flag, consumer CTAs count from shared memory.
                           Other kernels treat FUSED as AUTO; a window too small for two units, or a
                           record longer than a unit, falls back to ZC. */
  BK_GATHER_ADDR = 6    /* the paper's own stages 1-3 (§IV.A):
                           stage 1 on the GPU generates every element address of every lane (elements
                           of addr_elem_bytes), recognises per-lane base + stride patterns online
                           (T = 8 buffered addresses, periods <= 4, verify, fall back to explicit
                           addresses; BK_FLAG_NO_PATTERNS: always explicit) and writes descriptors +
                           explicit addresses into pinned host memory; the host pool assembles each
                           lane's bytes from them in the warp-tile layout; one DMA H2D. Same staged
                           bytes as every other mode. Never graph-replayed (host work per chunk). */
} bk_gather_mode;

typedef struct bk_config {
  uint32_t struct_size;   /* = sizeof(bk_config) */
  int32_t device;         /* CUDA ordinal the context binds to */
  uint64_t window_bytes;  /* device working-set cap for ALL streaming buffers (slots, offsets
                             slices, lane tables); 0 = 2 GiB. Resident aggregates are outside it. */
  uint32_t n_slots;       /* ring depth N >= 2 ("at minimum two"); 0 = 4 */
  uint32_t gather_mode;   /* bk_gather_mode */
  uint64_t chunk_bytes;   /* accessed (payload) bytes per chunk; 0 = auto (fits a slot, >= ~32 chunks) */
  uint32_t lanes;         /* lanes (compute threads) per chunk, multiple of 32; 0 = auto */
  uint32_t host_threads;  /* CPU-assembly pool size (BK_GATHER_CPU / HYBRID); 0 = all hardware threads */
  uint64_t record_size;   /* fixed record length when record_offsets == NULL */
  uint32_t flags;         /* BK_FLAG_* */
  uint32_t lane_bytes;    /* target accessed bytes per lane when lanes == 0; 0 = the kernel's default */
  uint32_t zc_share_pm;   /* HYBRID: 0 = adaptive split (a chunk is gathered zero-copy whenever fewer
                             zero-copy chunks are in flight than max(1, min(n_slots-1, round(t_pack /
                             t_zc))) of the measured per-chunk host-packing and gather times, and
                             every chunk is when packing one costs more than n_slots gathers); else
                             per-mille of chunks gathered zero-copy, deterministic: chunk i is zero-copy
                             iff floor((i+1)s) > floor(i s). Zero-copy chunks run one at a time on their
                             own stream, concurrently with the DMAs of host-packed chunks */
  uint32_t addr_elem_bytes; /* BK_GATHER_ADDR: bytes read per generated address (1, 2, 4, 8, 16); every
                             accessed extent (or fixed record) length must be a multiple. 0 = the
                             largest such power of two <= 8 (1 for whole variable-length records) */
} bk_config;

#define BK_FLAG_PROFILE 1u  /* time every stage of every chunk with CUDA events (bk_stats.ms_*); implies
                               eager issue (no CUDA-graph replay: graph event nodes carry no timestamps) */
#define BK_FLAG_BASELINE_DBUF 2u  /* run the paper's GPU double-buffering baseline instead (P:329-339,
                                     P:994-996): raw whole-record chunks into 2 buffers (window/2 each)
                                     on 2 streams, kernel over contiguous per-thread record ranges.
                                     BK_K_WORDCOUNT, BK_K_GREP, BK_K_GROUPBY and BK_K_KMEANS (no cid write-back:
                                     BK_E_UNSUPPORTED) only; results identical. */
#define BK_FLAG_NO_GRAPH 8u  /* issue every pipeline eagerly instead of capturing/replaying a CUDA graph
                               (ZC / DENSE pipelines are otherwise captured on their first run per
                               kernel, parameters and plan, and replayed by later runs) */
#define BK_FLAG_TEST_DELAYS 16u  /* test only: random spin kernels before every stage on every stream and
                                   host sleeps before CPU assembly, to expose missing ordering */
#define BK_FLAG_BASELINE_SBUF 4u  /* the single-buffer variant: one buffer of the whole window,
                                     copy then compute, no overlap */
#define BK_FLAG_TRACE 128u  /* record every kernel and copy of a run with CUPTI activity records (libcupti
                               loaded at run time; BK_E_UNSUPPORTED without it) and derive the bk_stats
                               stage times / overlap from them — unlike BK_FLAG_PROFILE the run keeps its
                               CUDA-graph replay, so the stats describe the timed pipeline */
#define BK_FLAG_NO_PATTERNS 64u  /* BK_GATHER_ADDR: no pattern recognition, every element address is sent
                                    (the "addresses" column of the paper's Table II) */
#define BK_FLAG_KEEP_OUTPUTS_PINNED 32u  /* caller-owned per-record output arrays that bk_run writes by DMA
                                     (bk_out_kmeans.cid, bk_out_partition.out_records, bk_out_kmer.kmer /
                                     .count) are page-locked (cudaHostRegister) by bk_run. Default: only for
                                     the duration of that bk_run (each run pays the registration, ~0.1 s per
                                     GiB). With this flag the registration is cached across runs (at most eight
                                     arrays, oldest released first) and released by bk_unpin_outputs or
                                     bk_destroy: the caller must keep such arrays allocated until then. */

typedef struct bk_ctx bk_ctx;

/* Allocates the context, its streams, events and the staging ring (window_bytes) on
 * cfg->device. *out_ctx is owned by the caller and freed by bk_destroy. */
BK_API int bk_create(const bk_config* cfg, bk_ctx** out_ctx);

/* Maps a host data set (P:355-360 streamingMap). host_ptr[0..nbytes) and, if given,
 * record_offsets[0..n_records) are BORROWED until bk_destroy or the next registration.
 * record_offsets: u64 record start offsets relative to host_ptr, off[0] == 0, non-decreasing,
 * each <= nbytes; record i = [off[i], off[i+1]) with off[n] := nbytes; empty records are legal.
 * record_offsets == NULL: fixed records of cfg.record_size bytes (nbytes % record_size == 0,
 * n_records must equal nbytes / record_size). Memory is pinned ONCE here (cudaHostRegister,
 * mapped + portable, + read-only where the device supports it and host_ptr and nbytes are multiples
 * of 4 KiB so that the registration owns its pages: libbk never writes the data set)
 * unless already pinned; pre-pinned memory is left as is.
 * Validation is O(n) once: BK_E_INVAL on malformed offsets. */
BK_API int bk_register_segments(bk_ctx* ctx, const void* host_ptr, uint64_t nbytes,
                         const uint64_t* record_offsets, uint64_t n_records);

/* Runs built-in kernel `kernel_id` over every registered record through the pipeline.
 * Ordered after prior work on `stream`; returns when `out` is valid (blocking) and also
 * records completion on `stream`. `out` points to the kernel's caller-owned in/out struct
 * (bk_out_*), whose first two fields are {struct_size, kernel_id}; struct_size must equal the
 * sizeof of that kernel's struct (BK_E_INVAL), an unknown kernel_id is BK_E_UNSUPPORTED.
 * The calling thread's current CUDA device is left unchanged. */
BK_API int bk_run(bk_ctx* ctx, int kernel_id, void* stream, void* out);

/* NULL-safe. Unpins what bk_register_segments pinned (and any output arrays kept pinned under
 * BK_FLAG_KEEP_OUTPUTS_PINNED), frees device memory. */
BK_API int bk_destroy(bk_ctx* ctx);

/* Releases the output-array registrations cached under BK_FLAG_KEEP_OUTPUTS_PINNED, after which
 * the caller may free those arrays. BK_E_INVAL on NULL. */
BK_API int bk_unpin_outputs(bk_ctx* ctx);

BK_API const char* bk_strerror(int status);
BK_API const char* bk_last_error(void);

/* ---- per-kernel in/out structs (host pointers unless stated) ---- */
typedef struct bk_out_header { uint32_t struct_size; int32_t kernel_id; } bk_out_header;

/* Result arrays of the aggregating kernels (word count, group-by, k-means, k-mers) may be HOST or
 * DEVICE pointers (device memory of the context's GPU): libbk copies with unified addressing, so a
 * multi-GPU caller can point them at the buffers its NCCL collectives reduce in place (SURVEY
 * §8(e)) with no host round trip. Host arrays need not be pinned. When every array of a word-count
 * or k-mer result is reachable by kernels — device memory, caller-pinned host memory, or host
 * memory kept pinned (BK_FLAG_KEEP_OUTPUTS_PINNED) — the final kernel stores the results into them
 * directly (over PCIe for host memory) instead of staging them in HBM for a copy after the run. */
typedef struct bk_out_wordcount {
  bk_out_header h;
  uint64_t table_slots;     /* in: device hash-table slots (power of two); 0 = 2^20 */
  uint64_t cap;             /* in: capacity of the arrays below */
  uint64_t* word_off;       /* out: offset (rel. host_ptr) of one occurrence of each distinct word */
  uint32_t* word_len;       /* out: its length */
  uint64_t* word_count;     /* out: its count (unordered; compare as a multiset) */
  uint64_t n_words;         /* out: distinct words (> cap -> BK_E_CAPACITY) */
  uint64_t total_words;     /* out */
  uint64_t* word_h1;        /* out, optional (NULL): the word's identity, two 64-bit hashes of its bytes */
  uint64_t* word_h2;        /*   and length — equal across GPUs, the key of the multi-GPU merge (bk_merge_counts) */
} bk_out_wordcount;

typedef struct bk_out_grep {
  bk_out_header h;
  const uint8_t* pattern;   /* in: <= 32 bytes; empty matches every record */
  uint32_t pattern_len;
  uint32_t _pad;
  uint64_t first_index;     /* in: added to every index (the shard's first global record) */
  uint64_t cap;             /* in: capacity of idx */
  uint64_t* idx;            /* out: ascending matching record indices */
  uint64_t n_match;         /* out (> cap -> BK_E_CAPACITY) */
} bk_out_grep;

typedef struct bk_out_kmeans {
  bk_out_header h;
  const float* centroids;   /* in: K x 16 fp32 */
  uint32_t K;               /* in: 1..256 */
  uint32_t _pad;
  uint64_t first_index;     /* in: global index of record 0 (checksum) */
  uint64_t* count;          /* out: K */
  double* sum;              /* out: K x 16 */
  uint64_t chk;             /* out: sum_i mix64((i<<8) ^ cid_i) mod 2^64 */
  int32_t* cid;             /* out, optional (NULL): n_records cluster ids written back to the host
                               (P:563-572 writes to mapped data): per chunk into the slot,
                               then DMA'd on a D2H stream (page-locked per run, or cached with
                               BK_FLAG_KEEP_OUTPUTS_PINNED) */
} bk_out_kmeans;

typedef struct bk_out_partition {
  bk_out_header h;
  uint32_t n_buckets;       /* in: power of two, 1..4096 */
  uint32_t _pad;
  uint64_t* out_records;    /* out: n_records x 16 B, chunk-major runs, each chunk bucket-sorted and stable */
  uint64_t* chunk_counts;   /* out: n_chunks x n_buckets run lengths */
  uint64_t chunk_cap;       /* in: capacity of chunk_counts in chunks */
  uint64_t n_chunks;        /* out */
  uint64_t* bucket_count;   /* out: n_buckets totals */
} bk_out_partition;

typedef struct bk_out_groupby {
  bk_out_header h;
  uint32_t G;               /* in: number of keys (dense 0..G-1), 1..8192 (else BK_E_INVAL) */
  uint32_t _pad;
  uint64_t* count;          /* out: G */
  uint64_t* qty;            /* out: G */
  double* amount;           /* out: G */
} bk_out_groupby;

typedef struct bk_out_layout {
  bk_out_header h;
  uint32_t n_ext;           /* in: 0 = whole record, else extents (<= 8) */
  uint32_t ext_off[8];
  uint32_t ext_len[8];
  uint64_t chunk;           /* in: which chunk to dump */
  uint8_t* stage;           /* out: staged bytes (stage_cap) */
  uint64_t stage_cap;
  uint64_t* lane_first;     /* out: lanes entries each (lane_cap) */
  uint64_t* lane_nrec;
  uint64_t* lane_bytes;
  uint64_t lane_cap;
  uint64_t stage_size;      /* out */
  uint32_t lanes;           /* out */
  uint32_t _pad;
  uint64_t chunk_lo, chunk_hi, n_chunks; /* out */
} bk_out_layout;

typedef struct bk_out_kmer {
  bk_out_header h;
  uint32_t k;               /* in: 1..31 */
  uint32_t seq_off;         /* in: sequence field offset in every record */
  uint32_t seq_len;         /* in: sequence field length, a multiple of 16 */
  uint32_t _pad;
  uint64_t table_slots;     /* in: device table slots (power of two); 0 = 2^24 */
  uint64_t cap;             /* in: capacity of kmer / count */
  uint64_t* kmer;           /* out: distinct k-mers, 2-bit packed (A=0 C=1 G=2 T=3), unordered. Device
                               memory, caller-pinned host memory, or host memory kept pinned
                               (BK_FLAG_KEEP_OUTPUTS_PINNED): the final flush kernel stores the results
                               itself (over PCIe for host memory); other host memory receives a copy after
                               the run. Both arrays are written up to min(cap, n_kmers) entries. */
  uint64_t* count;          /* out */
  uint64_t n_kmers;         /* out: distinct (> cap -> BK_E_CAPACITY) */
  uint64_t total;           /* out: k-mer occurrences */
} bk_out_kmer;

typedef struct bk_out_pattern {
  bk_out_header h;
  uint32_t n_ext;           /* in: access spec, 0 = whole record, else extents (<= 8) */
  uint32_t ext_off[8];
  uint32_t ext_len[8];
  uint32_t elem_bytes;      /* in: element size of the address stream (1 = every byte, 4 = fp32 ...) */
  uint32_t T;               /* in: temporary address buffer entries, 2..16 */
  uint32_t pmax;            /* in: longest stride period tried, 1..4 */
  uint32_t _pad;
  uint64_t chunk;           /* in: chunk whose per-lane results are dumped (UINT64_MAX: none) */
  int32_t* lane_p;          /* out (dump): per lane period, 0 = explicit addresses */
  int64_t* lane_strides;    /* out (dump): 4 per lane */
  uint64_t* lane_base;      /* out (dump): first address (offset in the data set) */
  uint64_t* lane_count;     /* out (dump): addresses generated */
  uint64_t lane_cap;        /* in: capacity of the dump arrays in lanes */
  uint32_t lanes;           /* out: lanes per chunk */
  uint32_t _pad2;
  uint64_t n_lanes, n_pattern_lanes, n_addresses, n_explicit_addresses; /* out: totals over all chunks */
  uint64_t address_bytes;   /* out: 8 B per address if every address were sent (the paper's addrBuf) */
  uint64_t pattern_bytes;   /* out: descriptors for pattern lanes + 8 B per explicit fallback address */
} bk_out_pattern;

typedef struct bk_stats {
  uint32_t struct_size;
  uint32_t gather_mode;       /* mode the last run used */
  uint64_t n_chunks;
  uint64_t chunk_budget;      /* accessed bytes per chunk */
  uint32_t lanes;             /* lanes per chunk */
  uint32_t n_slots;
  uint64_t slot_bytes;        /* device bytes per ring slot */
  uint64_t bytes_accessed;    /* sum of accessed bytes = algorithmic payload (I3) */
  uint64_t bytes_h2d;         /* payload bytes that crossed the link (DENSE: whole records) */
  uint64_t bytes_meta;        /* offsets slices shipped to the device */
  uint64_t bytes_padding;     /* staged - accessed (HBM only, never on the link; A9) */
  uint64_t bytes_d2h;
  uint64_t kernel_launches;   /* this library's kernel launches in the last run */
  double ms_run;              /* wall time of the last bk_run */
  double ms_register;         /* pin + validate time of the last registration */
  double ms_device;           /* CUDA-event time of the last run on its compute stream */
  double ms_h2d;              /* BK_FLAG_PROFILE: summed per-chunk busy time of the H2D copies */
  double ms_addrgen;          /*   ... of stage 1 (address generation) */
  double ms_gather;           /*   ... of stage 2 (+3 in ZC mode): gather / re-layout kernels */
  double ms_compute;          /*   ... of stage 4 (compute kernels) */
  uint64_t n_gather;          /*   number of gather launches timed */
  uint64_t n_chunks_cpu;      /* chunks assembled by the host pool (CPU / HYBRID) */
  double ms_cpu_gather;       /* host time spent assembling them */
  double ms_xfer_busy;        /* BK_FLAG_PROFILE: union of the transfer intervals (DMA copies, zero-copy gathers) */
  double ms_compute_busy;     /*   union of the compute-kernel intervals */
  double ms_overlap;          /*   length of their intersection (copy/compute overlap) */
  double ms_zc;               /* BK_FLAG_PROFILE: busy time of the zero-copy gathers alone (stages 2+3 over PCIe) */
  uint64_t n_zc;              /*   number of zero-copy gather launches timed */
  double ms_relayout;         /*   busy time of the HBM -> HBM interleave kernels (DENSE raw chunks, packed CPU chunks) */
  uint64_t n_relayout;        /*   number of interleave launches timed */
  uint64_t n_chunks_zc;       /* chunks gathered zero-copy in the last run */
  uint64_t bytes_zc;          /* accessed bytes those chunks pulled over PCIe */
  uint64_t records_zc;        /* records in those chunks */
  double ms_d2h;              /* BK_FLAG_PROFILE: busy time of the device->host write-back copies (partitioned
                                 chunks, k-means cluster ids); counted in ms_xfer_busy */
  uint64_t n_d2h;             /*   number of write-back copies timed */
  uint64_t n_units;           /* BK_GATHER_FUSED: units streamed through the shared-memory ring */
  uint32_t unit_bytes;        /*   unit capacity in bytes (UB) */
  uint32_t fused_grid;        /*   persistent CTAs (one per SM) */
  uint32_t fused_loaders;     /*   of which loaders (stages 1-3) */
  uint32_t fused_ring_slots;  /*   HBM ring slots (R x slot <= window_bytes) */
  double fused_wait_frac;     /*   BK_FLAG_PROFILE: consumers' share of time waiting for a unit's flag */
  double fused_compute_frac;  /*   ... computing (stage 1 ranges + stage 4) while loaders stream later units */
  double fused_loader_wait_frac; /* loaders' share of time waiting for a free ring slot */
  uint64_t bytes_addr;        /* BK_GATHER_ADDR: address information the GPU wrote to host memory (48-B lane
                                 descriptors + 8 B per explicit address + 8 B per chunk) */
  uint64_t n_addr_lanes;      /*   lanes that generated addresses */
  uint64_t n_pattern_lanes;   /*   ... of which sent a verified pattern instead of their addresses */
  uint64_t n_addresses;       /*   element addresses generated */
  uint64_t n_explicit_addr;   /*   ... of which sent explicitly */
  uint32_t addr_elem_bytes;   /*   element size used */
  uint32_t _pad_addr;
  double ms_addr_wait;        /*   host time waiting for stage 1's address information */
  double ms_trace_span;       /* BK_FLAG_TRACE: first kernel/copy start to last end of the run (device) */
  uint64_t n_trace_records;   /*   kernels + copies + memsets traced */
  uint32_t graph_issue;       /* how the run's device work was issued: 0 eager (BK_FLAG_NO_GRAPH /
                                 PROFILE, host work per chunk, or outputs page-locked for this run only),
                                 1 captured as a CUDA graph and launched, 2 a cached graph replayed */
  uint32_t _pad_graph;
} bk_stats;

BK_API int bk_get_stats(const bk_ctx* ctx, bk_stats* s);

/* ---- user kernels over the staged chunks (the paper's general programming model) -------------
 * BigKernel's promise is that ANY data-parallel kernel over a record-partitioned host array runs
 * out of core without programmer-managed buffers: the programmer states
 * which bytes of a record the kernel touches (the access spec, what BigKernel's address
 * generation derives from the kernel's code) and writes the kernel against the
 * staged, interleaved layout. bk_run_user runs stages 1-3 exactly as for the built-in kernels and
 * calls back, once per chunk, so that the caller enqueues its own stage-4 kernel. */
typedef struct bk_access {
  uint32_t struct_size;     /* = sizeof(bk_access) */
  uint32_t n_ext;           /* 0 = the whole record; else 1..8 extents, in access order (duplicates
                               and overlaps allowed: every listed byte is staged) */
  uint32_t ext_off[8];      /* extent offset relative to the record start */
  uint32_t ext_len[8];      /* extent length; every record must contain every extent (BK_E_INVAL) */
  uint32_t lane_bytes;      /* target accessed bytes per lane (compute thread); 0 = 256 */
  uint32_t _reserved;
} bk_access;

/* One staged chunk, as seen by the caller's stage-4 kernel. All pointers are DEVICE pointers,
 * valid for work enqueued on the callback's stream during the callback; libbk recycles the slot
 * once that work has completed. Layout: lane t (0 <= t < lanes) owns records
 * [lanes_desc[t].first, +nrec) of the data set; its accessed bytes, concatenated in record order
 * then access order, are staged as 16-B words, word k at
 *   stage + tile_base[t / 32] + (k * 32 + t % 32) * 16,
 * zero-padded to the tile's longest lane. */
typedef struct bk_lane { uint64_t first; uint32_t nrec; uint32_t nbytes; } bk_lane;
typedef struct bk_chunk_view {
  uint32_t struct_size;       /* = sizeof(bk_chunk_view) */
  uint32_t lanes;             /* L, a multiple of 32 (tiles = L / 32) */
  uint64_t chunk_index;       /* 0 .. n_chunks-1; chunks may be computed concurrently, in any order */
  uint64_t n_chunks;
  uint64_t first_record;      /* the chunk is records [first_record, first_record + n_records) */
  uint64_t n_records;
  const uint8_t* stage;       /* device: the warp tiles */
  const bk_lane* lane_desc;   /* device: L lane descriptors */
  const uint64_t* tile_base;  /* device: L/32 + 1 tile offsets (tile_base[L/32] = staged bytes) */
  const uint64_t* offsets;    /* device: record start offsets (relative to host_ptr) of the chunk's
                                 records, n_records entries, when the access is whole variable-length
                                 records; NULL otherwise (records then have a fixed accessed size) */
  uint64_t end_offset;        /* end of the chunk's last record (relative to host_ptr) */
} bk_chunk_view;

/* Called on the bk_run_user thread once per chunk, after that chunk's stages 1-3 are ordered on
 * `stream` (a cudaStream_t): enqueue stage-4 work on `stream` only, do not synchronise it, and
 * return 0. A non-zero return aborts the run with BK_E_INVAL (work already enqueued completes). */
typedef int (*bk_chunk_fn)(const bk_chunk_view* view, void* stream, void* user);

/* Streams the registered data set through stages 1-3 under `access` and calls `fn` per chunk;
 * ordered after prior work on `stream`, returns when every chunk's enqueued work has completed.
 * Gather mode, window and ring depth come from the context's bk_config (AUTO: DENSE for whole
 * records, HYBRID for sparse extents). Errors: BK_E_INVAL (NULL fn / access, bad extents, fn
 * returned non-zero), BK_E_STATE (nothing registered), BK_E_RANGE (a record's accessed bytes exceed
 * a chunk), BK_E_CUDA. Not available with BK_FLAG_BASELINE_* (BK_E_UNSUPPORTED). */
BK_API int bk_run_user(bk_ctx* ctx, const bk_access* access, bk_chunk_fn fn, void* user, void* stream);

/* ---- multi-GPU merge of count tables (SURVEY §8(e), C1 word count / f4 k-mers) ----------------
 * Per-GPU tables are all-gathered (NCCL over NVLink, by the caller) into one device buffer; this
 * merges them by key on the context's GPU. All pointers are DEVICE pointers on that GPU except
 * seg_rows (host).
 *   rows       n_seg segments of seg_stride rows each (segment r = rank r's table, padded to the
 *              longest); segment r holds seg_rows[r] <= seg_stride valid rows. A row is row_u64
 *              u64 words: words [0, key_u64) are its key, word count_col (>= key_u64) its count.
 *   out        cap rows of row_u64 words: one per distinct key, the count the sum over all rows of
 *              that key, every other word copied from its first row in (segment, row) order —
 *              e.g. the lowest rank's occurrence offset. Rows are in unspecified order.
 *   *n_out     (host) distinct keys; > cap: BK_E_CAPACITY, out holds cap of them.
 * Ordered after `stream`; returns when out and *n_out are valid. BK_E_INVAL: NULL pointers,
 * key_u64 == 0, count_col < key_u64 or >= row_u64, row_u64 > 16, seg_rows[r] > seg_stride. */
BK_API int bk_merge_counts(bk_ctx* ctx, const uint64_t* rows, uint32_t n_seg, uint64_t seg_stride,
                           const uint64_t* seg_rows, uint32_t row_u64, uint32_t key_u64, uint32_t count_col,
                           uint64_t* out, uint64_t cap, uint64_t* n_out, void* stream);

/* ---- user address generation (the paper's address mode with a caller-written stage 1) -----------
 * BigKernel derives stage 1 from the kernel's own address computations; here the caller
 * supplies that slice as a generator kernel. Per chunk libbk plans the lanes (contiguous record
 * ranges balanced under `bound`, the access spec that bounds what the generator may touch), calls
 * `gen` to enqueue the caller's kernel, which writes lane t's element addresses (byte offsets into
 * the registered data set, in the order its stage-4 kernel will consume them) at
 * addr[addr_base[t] + k], k < lane_desc[t].nbytes / elem_bytes, and the number written at
 * addr_count[t] (counts start at 0). Then libbk runs the online pattern recogniser over those
 * addresses, ships patterns / explicit addresses to the host, assembles the lanes (elem_bytes read
 * at each address) in the warp-tile layout, DMAs them and calls `fn` (bk_run_user's stage-4
 * callback) with lane_desc[t].nbytes = count x elem_bytes. Addresses outside the data set:
 * BK_E_INVAL. All pointers in the view are DEVICE pointers valid for work enqueued on `stream`. */
typedef struct bk_addr_view {
  uint32_t struct_size;       /* = sizeof(bk_addr_view) */
  uint32_t lanes;
  uint64_t chunk_index, n_chunks, first_record, n_records;
  const bk_lane* lane_desc;   /* lane t owns records [first, first + nrec); nbytes = its capacity in bytes */
  const uint64_t* offsets;    /* record start offsets of the chunk's records (n_records), variable-length
                                 records; NULL for fixed records (record r starts at r * record_size) */
  uint64_t end_offset;        /* end of the chunk's last record */
  uint64_t* addr;             /* out: element addresses, lane t's at addr[addr_base[t] + k] */
  const uint64_t* addr_base;  /* lanes entries */
  uint32_t* addr_count;       /* out: lanes entries, addresses lane t wrote */
  uint32_t elem_bytes;
  uint32_t _pad;
} bk_addr_view;
typedef int (*bk_addr_fn)(const bk_addr_view* view, void* stream, void* user);

/* Ordered after `stream`; returns when every chunk's stage-4 work has completed. Always address
 * mode (cfg.gather_mode is ignored; BK_FLAG_NO_PATTERNS applies). Errors as bk_run_user, plus
 * BK_E_INVAL for a generator address outside the data set or a count above the lane's capacity. */
BK_API int bk_run_user_addr(bk_ctx* ctx, const bk_access* bound, bk_addr_fn gen, void* gen_user, bk_chunk_fn fn,
                            void* user, void* stream);

/* ABI self-check for bindings: writes sizeof of bk_config, bk_out_wordcount, bk_out_grep,
 * bk_out_kmeans, bk_out_partition, bk_out_groupby, bk_out_layout, bk_stats, bk_out_pattern,
 * bk_out_kmer, bk_access, bk_chunk_view, bk_addr_view (in that order, up to n entries) and returns
 * BK_ABI_VERSION. Needs no GPU. */
BK_API int bk_abi_sizes(uint32_t* sizes, int n);

/* ---- C4 output in bucket-major order (host side, optional; SURVEY §8(d) C4 "a bucket-major
 * materialised copy is an optional, separately timed host pass") -------------------------------
 * BK_K_PARTITION leaves its result as chunk-major runs (each chunk bucket-sorted and stable,
 * chunk_counts[c * n_buckets + b] records of bucket b in chunk c), which is already the stable
 * partition up to a re-ordering of whole runs (chunks ascend in record order). This copies the runs
 * into the O4 order (bucket, original index) of PAPER.md's data-parallel partition (P:16-17 via
 * SURVEY O4): dst[bucket_start[b] + k] = k-th record of bucket b, taking chunk 0's run of b, then
 * chunk 1's, and so on.
 *   out_records   n x 16 B, the chunk-major runs bk_run wrote (n = sum of chunk_counts)
 *   chunk_counts  n_chunks x n_buckets, row-major, as bk_run wrote them
 *   bucket_start  n_buckets destination indices (records) of each bucket's first record, or NULL for
 *                 the local exclusive scan of the bucket totals (dst then holds exactly n records).
 *                 Multi-GPU: pass the global offsets of this rank's records (merge.py
 *                 merge_partition_offsets) so every rank fills its disjoint share of one array.
 *   dst           destination, 16-B records, caller-owned, must not overlap out_records
 *   threads       host threads (0 = all cores)
 * Pure host code, no CUDA call: it may run while the GPU streams the next data set. Returns BK_OK,
 * or BK_E_INVAL on NULL pointers, n_buckets == 0 or n_chunks * n_buckets overflow. */
BK_API int bk_partition_materialize(const void* out_records, const uint64_t* chunk_counts, uint64_t n_chunks,
                                    uint32_t n_buckets, const uint64_t* bucket_start, void* dst, uint32_t threads);

#ifdef __cplusplus
}
#endif
#endif
