// bk_internal.cuh — shared device/host definitions of libbk (product path only; never the oracle).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace bk {

constexpr int kWarp = 32;
constexpr int kMaxExt = 8;

// Lane descriptor written by stage 1 (address generation), 16 B. Lane t owns records
// [first, first + nrec) of the chunk (each thread a contiguous record range) and
// nbytes accessed bytes, staged as ceil(nbytes/16) 16-byte words.
struct LaneDesc {
  uint64_t first;
  uint32_t nrec;
  uint32_t nbytes;
};

// Access spec of a kernel: the bytes of each record its compute touches.
struct Access {
  uint32_t whole;        // 1: every byte of the record
  uint32_t n_ext;        // else: extents relative to the record start, in access order
  uint32_t ext_off[kMaxExt];
  uint32_t ext_len[kMaxExt];
  uint32_t E;            // sum of ext_len (accessed bytes per record) when !whole
  uint64_t rec_size;     // fixed record length, 0 = variable (offsets)
};

// One chunk = records [lo, hi) (whole records only, A3).
struct Chunk {
  uint64_t lo, hi;
  uint64_t base_byte;    // start offset of record lo (relative to the data set)
  uint64_t end_byte;     // end offset of record hi-1
  uint32_t L;            // lanes
  uint32_t ntiles;       // L / 32
  uint64_t accessed;     // A(lo, hi)
  // gather source bounds, in bytes around src: [src - guard_lo, src + guard_hi) is readable
  // (zero-copy: the registered data set; DENSE: the raw slot). Aligned 16-B words that would
  // straddle a bound are assembled from in-range bytes only.
  uint64_t guard_lo, guard_hi;
};

// Device error bits (sticky, read back at the end of bk_run).
enum : int {
  kErrStageOverflow = 1,
  kErrTableFull = 2,
  kErrKeyRange = 4,
  kErrWordTooLong = 8,
  kErrOutOverflow = 16,
  kErrFusedTimeout = 32,   // a persistent kernel's producer/consumer wait exceeded its limit
};

// SM count of the current device (queried once per device, then cached): grids are sized in
// multiples of it instead of a hard-coded 148.
inline int device_sms() {
  static int cache[64] = {};
  int d = 0;
  if (cudaGetDevice(&d) != cudaSuccess || d < 0 || d >= 64) return 148;
  if (!cache[d]) {
    int n = 0;
    if (cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, d) != cudaSuccess || n <= 0) n = 148;
    cache[d] = n;
  }
  return cache[d];
}

__host__ __device__ inline uint64_t mix64(uint64_t x) {
  x ^= x >> 30; x *= 0xbf58476d1ce4e5b9ULL;
  x ^= x >> 27; x *= 0x94d049bb133111ebULL;
  x ^= x >> 31;
  return x;
}

// ---- launchers (kernels_stage.cu) ----
// test-only: a one-thread kernel that spins `cycles` SM clocks (BK_FLAG_TEST_DELAYS)
void launch_spin(long long cycles, cudaStream_t s);
// Stage 1: lane plan + per-tile word counts, then tile bases (exclusive scan of 512*K_w).
// staged_sum accumulates the staged bytes of every chunk (padding statistics). meta_src (whole
// variable-length records only): the chunk's offsets in mapped host memory, read zero-copy and
// copied into `meta` on the way (no separate offsets DMA); nullptr = `meta` is already filled.
void launch_addrgen(const Chunk& c, const Access& a, const uint64_t* meta, LaneDesc* lanes,
                    uint32_t* tileK, uint64_t* tile_base, uint64_t stage_cap, int* err,
                    unsigned long long* staged_sum, cudaStream_t s, const uint64_t* meta_src = nullptr);
// Stage 2 (+3 when zero_copy: src is pinned, mapped host memory): gather the accessed bytes
// into warp tiles. src points at byte c.base_byte of the data set, same alignment mod 16.
void launch_gather(const Chunk& c, const Access& a, const uint8_t* src, const uint64_t* meta,
                   const LaneDesc* lanes, const uint64_t* tile_base, uint8_t* stage, uint64_t stage_cap,
                   int zero_copy, cudaStream_t s);

// ---- compute kernels (kernels_compute.cu) ----
struct WcEntry {            // 32 B open-addressing slot
  unsigned long long key1;  // 0 = empty
  unsigned long long key2;  // 0 = being published
  unsigned long long count;
  unsigned long long offlen; // occurrence offset (40 bits) | length (24 bits)
};
void launch_wc(const Chunk& c, const uint8_t* stage, const LaneDesc* lanes, const uint64_t* tile_base,
               const uint64_t* meta, uint64_t rec_size, WcEntry* table, uint64_t mask,
               unsigned long long* used, int* err, cudaStream_t s);
// C1 as one persistent launch (loader CTAs stream units into an HBM ring, consumer CTAs count):
// unit plan ub/uby (U+1 each, device), UB/UR bytes/records caps per unit; ready/done: R flags each,
// zeroed before the launch; prof optional (5 counters)
uint32_t wc_fused_slot_bytes(uint32_t UB, uint32_t UR);
size_t wc_fused_smem(uint32_t UB, uint32_t UR);
int wc_fused_grid();
uint32_t wc_fused_threads();
// DMA-fed variant: the copy engine fills K slots with batches of consecutive units (the host issues
// copy + stream-ordered flag write per batch); every CTA consumes
struct FusedDma {
  const uint32_t* ubatch;   // U: unit -> batch
  const uint64_t* bby;      // NB + 1: batch byte bounds
  const uint64_t* brec;     // NB + 1: batch record bounds
  const uint32_t* bunits;   // NB: units per batch
  uint32_t K;
  uint64_t bslot_bytes, btext;   // slot = [btext + 64 text][offsets]
  unsigned int* bcnt;       // K (zeroed)
};
cudaError_t launch_wc_fused(const uint8_t* data, uint64_t nbytes, const uint64_t* off, uint64_t rec_size,
                            const uint64_t* ub, const uint64_t* uby, uint32_t U, uint32_t UB, uint32_t UR, int grid,
                            uint32_t n_load, uint8_t* ring, uint32_t R, unsigned long long* ready,
                            unsigned long long* done, WcEntry* table, uint64_t mask, unsigned long long* used,
                            int* err, unsigned long long* prof, const FusedDma* dma, cudaStream_t s);
// double-buffering baseline (variant iv): raw chunk bytes start at absolute offset base_byte
void launch_dbuf_wc(const uint8_t* raw, const uint64_t* meta, uint64_t lo, uint64_t hi, uint64_t base_byte,
                    uint64_t end_byte, uint64_t rec_size, WcEntry* table, uint64_t mask, unsigned long long* used,
                    int* err, cudaStream_t s);
// distinct words -> (occurrence offset, length, count, key1, key2) rows; *total += every count
void launch_wc_compact(WcEntry* table, uint64_t slots, unsigned long long* n_out, unsigned long long* total,
                       uint64_t* off, uint32_t* len, uint64_t* cnt, uint64_t* h1, uint64_t* h2, uint64_t cap,
                       cudaStream_t s);

struct GrepParams {
  uint8_t pat[32];
  uint32_t plen;
  uint64_t first_index;
  uint64_t cap;
};
// three launches per chunk: per-tile counts + per-lane match masks, a one-block scan (reserves the
// chunk's run [base, base+n) of the match pool with atomicAdd on *cursor, writes chunk_run =
// {base, n} and each tile's output base), ordered write into the pool. Chunks may run
// concurrently; launch_grep_order then lays the runs out in chunk order. tilecnt / tilebase_out
// hold c.ntiles entries, lanemask c.L.
size_t grep_count_smem();
void launch_grep(const Chunk& c, const uint8_t* stage, const LaneDesc* lanes, const uint64_t* tile_base,
                 const GrepParams& p, uint32_t* tilecnt, uint32_t* lanemask, unsigned long long* cursor,
                 unsigned long long* tilebase_out, unsigned long long* chunk_run, uint64_t* out_idx, int* err,
                 int grid, bool tma, cudaStream_t s);
void launch_grep_order(const unsigned long long* runs, uint32_t C, const uint64_t* pool, uint64_t* out, uint64_t cap,
                       cudaStream_t s);

// tma: stage-4 reads through bulk copies into shared memory (tma.cuh); false: plain 16-B loads
// (chunks computed while zero-copy gathers run, profiles/r01_tma.md)
size_t groupby_smem(uint32_t G, bool tma);
void launch_groupby(const Chunk& c, const uint8_t* stage, const LaneDesc* lanes, const uint64_t* tile_base,
                    uint32_t G, unsigned long long* count, unsigned long long* qty, double* amount, int* err,
                    int grid, bool tma, cudaStream_t s);

size_t kmeans_smem(uint32_t K, bool tma);
void launch_kmeans(const Chunk& c, const uint8_t* stage, const LaneDesc* lanes, const uint64_t* tile_base,
                   const float* mu, uint32_t K, uint64_t first_index, unsigned long long* count, double* sum,
                   unsigned long long* chk, int32_t* cid_out, int grid, bool tma, cudaStream_t s);

cudaError_t configure_compute_kernels();

// ---- C4 partition (kernels_partition.cu): 4 launches per chunk ----
size_t partition_smem(uint32_t B);
uint32_t partition_blocks(const Chunk& c);
void launch_partition(const Chunk& c, const uint8_t* stage, const LaneDesc* lanes, const uint64_t* tile_base,
                      int bits, uint32_t* hist, uint32_t* colpre, unsigned long long* total,
                      unsigned long long* base, uint8_t* out, cudaStream_t s);
cudaError_t configure_partition_kernels();

// ---- the paper's double-buffering baseline (kernels_baseline.cu) ----
uint32_t dbuf_blocks();
void launch_dbuf_grep(const uint8_t* raw, const uint64_t* meta, uint64_t lo, uint64_t hi, uint64_t base_byte,
                      uint64_t end_byte, uint64_t rec_size, const GrepParams& p, uint32_t* blkcnt,
                      unsigned long long* running, unsigned long long* blkbase, uint64_t* out, cudaStream_t s);
void launch_dbuf_groupby(const uint8_t* raw, uint64_t lo, uint64_t hi, uint64_t base_byte, uint64_t rec_size,
                         uint32_t G, unsigned long long* count, unsigned long long* qty, double* amount, int* err,
                         cudaStream_t s);
void launch_dbuf_kmeans(const uint8_t* raw, uint64_t lo, uint64_t hi, uint64_t base_byte, uint64_t rec_size,
                        const float* mu, uint32_t K, uint64_t first_index, unsigned long long* count, double* sum,
                        unsigned long long* chk, cudaStream_t s);
cudaError_t configure_baseline_kernels();

// ---- f4: k-mer counting over DNA reads (kernels_kmer.cu) ----
struct KmerEntry {            // 16 B exact-key slot
  unsigned long long key;     // k-mer + 1 (0 = empty)
  unsigned long long count;
};
// two-phase counting (kernels_kmer.cu): the table as 2^rb regions of region_slots slots; phase A
// appends keys to per-region buckets (bbuf: 2^rb x bcap keys, bcur: 2^rb cursors, dirty: 2^rb flags,
// all zeroed), a flush counts each bucket into its region in shared memory; the final flush emits the
// distinct k-mers to out_kmer / out_cnt (n_out, zeroed) instead of writing the regions back
size_t kmer_flush_smem(uint64_t region_slots);
// phase A: k-mer keys -> 2^cb coarse bins (cb <= rb; cb == rb: the bins are the regions' buckets)
void launch_kmer_bin(const Chunk& c, const uint8_t* stage, const LaneDesc* lanes, const uint64_t* tile_base,
                     uint32_t k, uint32_t seq_words, KmerEntry* table, uint32_t rb, uint32_t cb, uint64_t region_slots,
                     unsigned long long* gbuf, unsigned int* gcur, uint32_t gcap, unsigned char* dirty,
                     unsigned long long* total, int* err, cudaStream_t s);
// flush, first half (cb < rb): coarse bins -> region buckets, coarse cursors reset (cdone: 2^cb, zeroed)
void launch_kmer_split(const unsigned long long* cbuf, unsigned int* ccur, uint32_t ccap, unsigned int* cdone,
                       uint32_t rb, uint32_t cb, unsigned long long* fbuf, unsigned int* fcur, uint32_t fcap,
                       KmerEntry* table, uint64_t region_slots, unsigned char* dirty, int* err, cudaStream_t s);
void launch_kmer_flush(KmerEntry* table, uint32_t rb, uint64_t region_slots, const unsigned long long* bbuf,
                       unsigned int* bcur, uint32_t bcap, unsigned char* dirty, int final_flush, uint64_t* out_kmer,
                       uint64_t* out_cnt, uint64_t ocap, unsigned long long* n_out, int* err, cudaStream_t s);
cudaError_t configure_kmer_kernels();

// ---- multi-GPU merge of count tables (kernels_merge.cu): rows of row_u64 words, key = words
// [0, key_u64), count at count_col; owner/cnt: `slots` (power of two) scratch entries each
cudaError_t launch_merge_counts(const uint64_t* rows, uint32_t n_seg, uint64_t seg_stride, const uint64_t* seg_rows,
                                uint32_t row_u64, uint32_t key_u64, uint32_t count_col, unsigned long long* owner,
                                unsigned long long* cnt, uint64_t slots, uint64_t* out, uint64_t cap,
                                unsigned long long* n_out, int* err, cudaStream_t s);

// ---- stage 1 in address mode (kernels_addr.cu, BK_GATHER_ADDR) ----
// One lane's address information as the host receives it (48 B): the element addresses are
// base, base + stride[0], + stride[1], ... (strides repeat with period p) when p > 0; when p == 0
// they are listed explicitly (count of them, in the chunk's compacted explicit-address buffer).
struct AddrDesc {
  uint64_t base;
  int64_t stride[4];
  uint32_t count;   // element addresses of the lane
  int32_t p;        // period (1..4), 0 = explicit
};
// detect / verify per lane (descriptors to desc_host, mapped host memory), exclusive scan of the
// explicit counts (total to *total_host), explicit addresses to exp_dev then exp_host (mapped).
// user_addr != nullptr: addresses from a caller's generator (lane t: user_addr[user_base[t] + k],
// k < user_count[t]); the kernel then also sets lanes[t].nbytes and tileK (run launch_tile_scan after).
void launch_addr_stage1(const Chunk& c, const Access& a, const uint64_t* meta, LaneDesc* lanes, uint32_t* tileK,
                        uint32_t elem, uint32_t T, uint32_t pmax, int patterns, const uint64_t* user_addr,
                        const uint64_t* user_base, const uint32_t* user_count, AddrDesc* desc_host,
                        uint32_t* ecount, uint64_t* epos, uint64_t* exp_dev, uint64_t* exp_host,
                        uint64_t* total_host, cudaStream_t s);
// bk_run_user_addr: lane t's address capacity lanes[t].nbytes / elem (into tmp) and its exclusive
// scan base[t] (base[L] = total) — where the caller's generator writes lane t's addresses
void launch_lane_bases(uint32_t L, const LaneDesc* lanes, uint32_t elem, uint32_t* tmp, uint64_t* base,
                       cudaStream_t s);
// tile bases from the per-tile word counts (the last kernel of launch_addrgen), for lane plans
// whose byte counts were set after address generation
void launch_tile_scan(const uint32_t* tileK, uint32_t ntiles, uint64_t* tile_base, uint64_t stage_cap, int* err,
                      unsigned long long* staged_sum, cudaStream_t s);

// ---- online pattern recognition (kernels_pattern.cu, NEXT f2) ----
void launch_addr_patterns(const Chunk& c, const Access& a, const uint64_t* meta, const LaneDesc* lanes, uint32_t elem,
                          uint32_t T, uint32_t pmax, int32_t* lane_p, int64_t* lane_strides, uint64_t* lane_base,
                          uint64_t* lane_count, unsigned long long* totals, int dump, cudaStream_t s);

}  // namespace bk
