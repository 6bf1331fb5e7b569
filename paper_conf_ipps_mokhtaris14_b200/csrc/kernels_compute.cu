// kernels_compute.cu — pipeline stage 4 (Fig. 3):
// the compute kernels read their lane's words from the staged warp tiles (one coalesced
// 512-B access per warp per word, the point of the interleaved layout) and
// reduce with warp-level aggregation and block-level shared-memory tables before touching
// global memory (north_star: warp shuffles + block-level atomics).
#include "bk_internal.cuh"
#include "tma.cuh"

#include <algorithm>

namespace bk {
namespace {

constexpr unsigned kFull = 0xffffffffu;

__device__ __forceinline__ uint4 lane_word(const uint8_t* tile, uint32_t k, int lane) {
  return __ldcs(reinterpret_cast<const uint4*>(tile + ((size_t)k * 32 + lane) * 16));
}

// ------------------------------------------------------------------------------------------
// C1 word count (centralized hash table).
// A word is a maximal run of non-delimiter bytes inside one record (reading A10/A19).
// Identity = (two independent 64-bit hashes, length); the table stores one occurrence offset
// so the host can recover the bytes.

__device__ __forceinline__ bool is_delim(uint32_t ch) { return ch == 0x20 || (ch - 0x09u) <= 4u; }

__device__ __noinline__ void wc_insert(WcEntry* table, uint64_t mask, unsigned long long key1, unsigned long long key2,
                                       unsigned long long offlen, unsigned long long cnt, unsigned long long* used,
                                       int* err) {
  uint64_t slot = key1 & mask;
  for (uint64_t probe = 0; probe <= mask; ++probe, slot = (slot + 1) & mask) {
    WcEntry* e = &table[slot];
    unsigned long long k = *reinterpret_cast<volatile unsigned long long*>(&e->key1);
    if (k == 0) {
      k = atomicCAS(&e->key1, 0ull, key1);
      if (k == 0) {  // claimed: publish occurrence, then key2
        e->offlen = offlen;
        __threadfence();
        atomicExch(&e->key2, key2);
        atomicAdd(&e->count, cnt);
        atomicAdd(used, 1ull);
        return;
      }
    }
    if (k == key1) {
      unsigned long long k2;
      while ((k2 = *reinterpret_cast<volatile unsigned long long*>(&e->key2)) == 0) {
      }
      if (k2 == key2) {
        atomicAdd(&e->count, cnt);
        return;
      }
    }
  }
  atomicOr(err, kErrTableFull);
}

// The common case of a global update: the word is already at its home slot. One 16-B L2 read of
// (key1, key2) and a fire-and-forget add; anything else takes the full probe/claim path.
__device__ __forceinline__ bool wc_home_hit(const ulonglong2 home, unsigned long long key1, unsigned long long key2) {
  return home.x == key1 && home.y == key2;
}

// Per-block shared-memory pre-aggregation (Zipf text: most occurrences hit a few hot words).
constexpr int kWcBlock = 128;   // 4 warps: small blocks spread a chunk's few lanes over more SMs
constexpr int kWcTab = 512;     // block table slots (a hot-word cache)
constexpr int kWcQ = 256;       // per-warp queue of finished words
constexpr int kWcProbes = 2;    // a crowded block-table slot sends the word to the global table

template <int NW, int Q>   // NW warps per block, Q queue entries per warp
struct WcSharedT {
  static constexpr int kQ = Q;
  unsigned long long k1[kWcTab], k2[kWcTab], ol[kWcTab];
  unsigned int cnt[kWcTab];
  unsigned long long qk1[NW][Q], qk2[NW][Q], qol[NW][Q];
};
using WcShared = WcSharedT<kWcBlock / 32, kWcQ>;

template <class SH>
__device__ void tab_insert(SH& sh, WcEntry* table, uint64_t mask, unsigned long long k1,
                           unsigned long long k2, unsigned long long ol, unsigned int cnt,
                           unsigned long long* used, int* err) {
  uint32_t s = (uint32_t)(k1 >> 20) & (kWcTab - 1);
  for (int p = 0; p < kWcProbes; ++p, s = (s + 1) & (kWcTab - 1)) {
    unsigned long long cur = atomicCAS(&sh.k1[s], 0ull, k1);
    if (cur == 0) {  // claimed: publish occurrence + key2 (readers spin until key2 != 0)
      sh.ol[s] = ol;
      __threadfence_block();
      atomicExch(&sh.k2[s], k2);
      atomicAdd(&sh.cnt[s], cnt);
      return;
    }
    if (cur == k1) {
      unsigned long long c2;
      while ((c2 = *reinterpret_cast<volatile unsigned long long*>(&sh.k2[s])) == 0) {
      }
      if (c2 == k2) {
        atomicAdd(&sh.cnt[s], cnt);
        return;
      }
    }
  }
  // block table crowded: go global
  const ulonglong2 home = __ldcg(reinterpret_cast<const ulonglong2*>(&table[k1 & mask]));
  if (wc_home_hit(home, k1, k2)) atomicAdd(&table[k1 & mask].count, (unsigned long long)cnt);
  else wc_insert(table, mask, k1, k2, ol, cnt, used, err);
}

// Insert the warp's n queued words, 32 at a time: finalise the identity here (every lane busy),
// merge duplicates within a round by match_any, insert into the block table.
template <class SH>
__device__ __noinline__ void wc_flush_queue(SH& sh, int w, int lane, int n, WcEntry* table,
                                            uint64_t mask, unsigned long long* used, int* err) {
  __syncwarp();
  for (int base = 0; base < n; base += 32) {
    const int i = base + lane;
    const bool v = i < n;
    unsigned long long k1 = 0, k2 = 0, ol = 0;
    if (v) {
      ol = sh.qol[w][i];
      const uint64_t len = ol & 0xffffff;
      k1 = mix64(sh.qk1[w][i] ^ (len * 0x9E3779B97F4A7C15ull)) | 1ull;
      k2 = mix64(sh.qk2[w][i] + len) | 1ull;
    }
    const unsigned m = __match_any_sync(kFull, k1) & __match_any_sync(kFull, k2);
    if (v && lane == __ffs(m) - 1) tab_insert(sh, table, mask, k1, k2, ol, __popc(m), used, err);
  }
  __syncwarp();
}

// Block table -> global table: thread `tid` of `nthreads` moves its slots (all home-slot reads in
// flight at once, then the adds), optionally clearing them for reuse.
template <class SH, int kPer>
__device__ __forceinline__ void wc_flush_block(SH& sh, int tid, int nthreads, WcEntry* table, uint64_t mask,
                                               unsigned long long* used, int* err, bool clear) {
  unsigned long long k1[kPer], k2[kPer];
  ulonglong2 home[kPer];
#pragma unroll
  for (int m = 0; m < kPer; ++m) {
    const int i = tid + m * nthreads;
    k1[m] = sh.k1[i];
    k2[m] = sh.k2[i];
    home[m] = k1[m] ? __ldcg(reinterpret_cast<const ulonglong2*>(&table[k1[m] & mask])) : make_ulonglong2(0, 0);
  }
#pragma unroll
  for (int m = 0; m < kPer; ++m) {
    const int i = tid + m * nthreads;
    if (!k1[m]) continue;
    if (wc_home_hit(home[m], k1[m], k2[m])) atomicAdd(&table[k1[m] & mask].count, (unsigned long long)sh.cnt[i]);
    else wc_insert(table, mask, k1[m], k2[m], sh.ol[i], sh.cnt[i], used, err);
    if (clear) { sh.k1[i] = 0; sh.k2[i] = 0; sh.cnt[i] = 0; }
  }
}


// kWcSub threads share one lane: sub-thread q owns the words that START in its quarter
// [q*span, (q+1)*span) of the lane's bytes and finishes its last word past the quarter end
// (classic parallel tokenisation; record boundaries from the offsets slice). Every 16-byte step
// is branch-free across the warp: a word ending at a byte takes a queue slot from a ballot, and
// its identity is finalised in the flush, so per-word work never rides on the per-byte path.
template <int kWcSub>  // sub-threads per lane
__global__ void __launch_bounds__(kWcBlock) k_wc(Chunk c, const uint8_t* __restrict__ stage,
                                                 const LaneDesc* __restrict__ lanes,
                                                 const uint64_t* __restrict__ tile_base,
                                                 const uint64_t* __restrict__ meta, uint64_t rec_size,
                                                 WcEntry* table, uint64_t mask, unsigned long long* used, int* err) {
  __shared__ WcShared sh;
  for (int i = threadIdx.x; i < kWcTab; i += blockDim.x) { sh.k1[i] = 0; sh.k2[i] = 0; sh.cnt[i] = 0; }
  __syncthreads();
  const uint32_t g = blockIdx.x * blockDim.x + threadIdx.x;
  const uint32_t t = g / kWcSub, q = g % kWcSub;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const unsigned lt = (1u << lane) - 1;
  const bool live_warp = (g & ~31u) / kWcSub < c.L;
  if (live_warp) {
    const bool live = t < c.L;
    LaneDesc d{0, 0, 0};
    if (live) d = lanes[t];
    const uint8_t* tile = live ? stage + tile_base[t >> 5] : stage;
    const int col = t & 31;
    auto rstart = [&](uint64_t r) -> uint64_t {
      if (rec_size) return r * rec_size;
      return r == c.hi ? c.end_byte : meta[r - c.lo];
    };
    const uint64_t lane_start = live ? rstart(d.first) : 0;
    const uint64_t rend = d.first + d.nrec;
    const uint32_t span = ((d.nbytes + kWcSub - 1) / kWcSub + 15) & ~15u;
    uint32_t pos0 = min(d.nbytes, q * span);
    const uint32_t range_end = min(d.nbytes, (q + 1) * span);
    // first record boundary strictly after pos0 (binary search over the lane's records)
    uint64_t r;
    {
      uint64_t lo = d.first + 1, hi = rend;
      while (lo < hi) {
        const uint64_t mid = (lo + hi) / 2;
        if (rstart(mid) - lane_start <= pos0) lo = mid + 1; else hi = mid;
      }
      r = lo;
    }
    const bool at_boundary = pos0 > 0 && r > d.first + 1 && rstart(r - 1) - lane_start == pos0;
    uint32_t next_b = r < rend ? (uint32_t)(rstart(r) - lane_start) : 0xffffffffu;
    auto byte_at = [&](uint32_t p) -> uint32_t {
      const uint4 v = lane_word(tile, p >> 4, col);
      const uint32_t j = p & 15;
      const uint32_t wd = j < 8 ? (j < 4 ? v.x : v.y) : (j < 12 ? v.z : v.w);
      return (wd >> (8 * (j & 3))) & 0xff;
    };
    // a word running into pos0 belongs to the previous sub-thread: start in "skip" state
    bool skip = live && q > 0 && pos0 < d.nbytes && !at_boundary && !is_delim(byte_at(pos0 - 1));
    bool in_word = false;
    uint64_t h1 = 0, h2 = 0;
    uint32_t wstart = 0, wlen = 0;
    int qn = 0;  // warp-uniform queue fill
    auto emit = [&](bool end) {
      const unsigned m = __ballot_sync(kFull, end);
      if (m) {
        if (end) {
          const uint64_t occ = lane_start + wstart;
          if (wlen >= (1u << 24) || occ >= (1ull << 40)) atomicOr(err, kErrWordTooLong);
          const int i = qn + __popc(m & lt);
          sh.qk1[w][i] = h1;
          sh.qk2[w][i] = h2;
          sh.qol[w][i] = (occ << 24) | wlen;
        }
        qn += __popc(m);
        if (qn > kWcQ - 32) {
          wc_flush_queue(sh, w, lane, qn, table, mask, used, err);
          qn = 0;
        }
      }
    };
    uint32_t k = pos0 >> 4;
    bool go = live && pos0 < range_end;
    while (__any_sync(kFull, go)) {
      const uint4 v = go ? lane_word(tile, k, col) : make_uint4(0, 0, 0, 0);
#pragma unroll
      for (int j = 0; j < 16; ++j) {
        const uint32_t pos = 16 * k + j;
        // a byte is ours while inside the quarter, or past it while finishing our last word
        const bool valid = go && pos >= pos0 && pos < d.nbytes && (pos < range_end || in_word || skip);
        const uint32_t wd = j < 8 ? (j < 4 ? v.x : v.y) : (j < 12 ? v.z : v.w);
        const uint32_t ch = (wd >> (8 * (j & 3))) & 0xff;
        const bool boundary = valid && pos == next_b;
        if (boundary) {
          do {  // several records may start here if some are empty
            ++r;
            next_b = r < rend ? (uint32_t)(rstart(r) - lane_start) : 0xffffffffu;
          } while (next_b == pos);
        }
        const bool delim = is_delim(ch);
        if (valid && (delim || boundary)) skip = false;
        const bool end = valid && in_word && (delim || boundary);
        emit(end);
        if (end) in_word = false;
        if (valid && !delim && !skip && (in_word || pos < range_end)) {
          if (!in_word) { in_word = true; wstart = pos; wlen = 0; h1 = 0xcbf29ce484222325ull; h2 = 0x84222325cbf29ce4ull; }
          h1 = (h1 ^ ch) * 0x100000001b3ull;
          h2 = (h2 + ch + 1) * 0x9E3779B97F4A7C15ull;
          h2 ^= h2 >> 29;
          ++wlen;
        }
      }
      ++k;
      go = go && 16 * k < d.nbytes && (16 * k < range_end || in_word || skip);
    }
    emit(in_word && live);
    if (qn) wc_flush_queue(sh, w, lane, qn, table, mask, used, err);
  }
  __syncthreads();
  // flush the block table: all of this thread's home-slot reads in flight at once, then adds
  wc_flush_block<WcShared, kWcTab / kWcBlock>(sh, threadIdx.x, kWcBlock, table, mask, used, err, false);
}

// The paper's double-buffering baseline for word count (variant iv): the
// same word identity and table as k_wc, but each thread scans a contiguous record range of the
// raw DMA'd chunk (AoS text) byte by byte and inserts every word into the global table
// directly — no lane layout, no block pre-aggregation.
__global__ void __launch_bounds__(256) k_dbuf_wc(const uint8_t* __restrict__ raw, const uint64_t* __restrict__ meta,
                                                 uint64_t lo, uint64_t hi, uint64_t base_byte, uint64_t end_byte,
                                                 uint64_t rec_size, WcEntry* table, uint64_t mask,
                                                 unsigned long long* used, int* err) {
  const uint64_t T = (uint64_t)gridDim.x * blockDim.x, t = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  const uint64_t n = hi - lo, a = lo + n * t / T, b = lo + n * (t + 1) / T;
  auto rstart = [&](uint64_t r) -> uint64_t {   // absolute data-set offset of record r
    if (!meta) return r * rec_size;
    return r == hi ? end_byte : meta[r - lo];
  };
  for (uint64_t r = a; r < b; ++r) {
    const uint64_t s0 = rstart(r), s1 = rstart(r + 1);
    uint64_t h1 = 0, h2 = 0, wstart = 0;
    uint32_t wlen = 0;
    for (uint64_t pos = s0; pos <= s1; ++pos) {
      const uint32_t ch = pos < s1 ? raw[pos - base_byte] : 0x20u;   // the record end is a delimiter
      if (is_delim(ch)) {
        if (wlen) {
          if (wlen >= (1u << 24) || wstart >= (1ull << 40)) atomicOr(err, kErrWordTooLong);
          const unsigned long long k1 = mix64(h1 ^ ((uint64_t)wlen * 0x9E3779B97F4A7C15ull)) | 1ull;
          const unsigned long long k2 = mix64(h2 + wlen) | 1ull;
          wc_insert(table, mask, k1, k2, (wstart << 24) | wlen, 1, used, err);
          wlen = 0;
        }
        continue;
      }
      if (!wlen) { wstart = pos; h1 = 0xcbf29ce484222325ull; h2 = 0x84222325cbf29ce4ull; }
      h1 = (h1 ^ ch) * 0x100000001b3ull;
      h2 = (h2 + ch + 1) * 0x9E3779B97F4A7C15ull;
      h2 ^= h2 >> 29;
      ++wlen;
    }
  }
}

// Occupied slots -> the result arrays, each drained slot zeroed. Each block compacts 1024 consecutive slots into shared memory
// (ballot + block scan, slot order), reserves its run with ONE atomic, and stores the run coalesced,
// so the stores are long contiguous runs per array — the result arrays may be the caller's mapped
// host memory, written over PCIe (a table is ~5% occupied: per-warp runs would be a few bytes each).
// h1 / h2 (the word's two hashes, for the multi-GPU merge) are written only when asked for.
constexpr int kCmpThreads = 256;
constexpr uint32_t kCmpSlots = 1024;   // slots per block

__global__ void __launch_bounds__(kCmpThreads) k_wc_compact(WcEntry* __restrict__ table, uint64_t slots,
                                                            unsigned long long* n_out, unsigned long long* total,
                                                            uint64_t* off, uint32_t* len, uint64_t* cnt, uint64_t* h1,
                                                            uint64_t* h2, uint64_t cap) {
  __shared__ uint64_t s_off[kCmpSlots], s_cnt[kCmpSlots], s_h1[kCmpSlots], s_h2[kCmpSlots];
  __shared__ uint32_t s_len[kCmpSlots];
  __shared__ unsigned s_warp[kCmpThreads / 32];
  __shared__ unsigned s_n;
  __shared__ unsigned long long s_base;
  const uint32_t tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  const uint64_t lo = (uint64_t)blockIdx.x * kCmpSlots, hi = min(slots, lo + kCmpSlots);
  if (tid == 0) s_n = 0;
  unsigned long long mine = 0;
  for (uint64_t i0 = lo; i0 < hi; i0 += kCmpThreads) {
    const uint64_t i = i0 + tid;
    WcEntry e{};
    if (i < hi) e = table[i];
    const bool occ = e.key1 != 0;
    const unsigned m = __ballot_sync(kFull, occ);
    if (lane == 0) s_warp[w] = __popc(m);
    __syncthreads();
    unsigned before = s_n, tot = 0;
    for (uint32_t q = 0; q < kCmpThreads / 32; ++q) {
      before += q < w ? s_warp[q] : 0u;
      tot += s_warp[q];
    }
    if (occ) {
      table[i] = WcEntry{};   // drained: the table is all zero for the next run (no memset)
      const unsigned p = before + __popc(m & ((1u << lane) - 1));
      s_off[p] = e.offlen >> 24;
      s_len[p] = (uint32_t)(e.offlen & 0xffffff);
      s_cnt[p] = e.count;
      s_h1[p] = e.key1;
      s_h2[p] = e.key2;
      mine += e.count;
    }
    __syncthreads();
    if (tid == 0) s_n += tot;
  }
  __syncthreads();
  const unsigned n = s_n;
  if (tid == 0) s_base = n ? atomicAdd(n_out, (unsigned long long)n) : 0ull;
  __syncthreads();
  const unsigned long long base = s_base;
  for (uint32_t j = tid; j < n; j += kCmpThreads) {
    const unsigned long long p = base + j;
    if (p >= cap) break;
    off[p] = s_off[j];
    len[p] = s_len[j];
    cnt[p] = s_cnt[j];
    if (h1) h1[p] = s_h1[j];
    if (h2) h2[p] = s_h2[j];
  }
  // total words: one atomic per warp
  for (int o = 16; o; o >>= 1) mine += __shfl_down_sync(kFull, mine, o);
  if (lane == 0 && mine) atomicAdd(total, mine);
}

// ------------------------------------------------------------------------------------------
// C1 word count as ONE persistent launch: BigKernel's single kernel ("a single kernel
// invocation"; Fig. 3: inside one launch, address-generation threads and compute threads
// are specialised and synchronise through flags, the buffers ring across iterations, P:546-561,
// P:790-860), specialised per CTA on sm_100a:
//   * LOADER CTAs (stages 1-3): per unit of whole records (planned on the host once per
//     registration, a1), copy the unit's record offsets and exactly its bytes from pinned, mapped
//     host memory (zero-copy, coalesced 16-B loads, every byte once) into a ring slot in HBM, then
//     publish the slot (release flag) — the paper's signal_dataReady;
//   * CONSUMER CTAs (stage 4): wait for a unit's flag (acquire), copy the slot into shared memory,
//     release the slot (the loader of unit u+R may refill it), derive each thread's byte range and
//     record boundaries from the offsets (stage 1's lane plan), tokenise and count (warp queue ->
//     block hot-word table -> global table, identities as k_wc).
// Why split by CTA (= by SM, one CTA per SM): an SM's global loads queue behind its own
// outstanding PCIe reads, which drain at that SM's share of the link (~0.35 GB/s): with zero-copy
// traffic in flight a hash-table load took tens of microseconds (ncu, r02c: 36% of warp samples on
// one unit-metadata load). Loader SMs only stream; consumer SMs never touch host memory.
// The HBM ring (R slots, R x slot <= window_bytes) is the device working set; ring order and the
// n - R reuse distance follow the paper's buffer-instance rule. Every spin has a
// %globaltimer limit (error flag instead of a hang).
constexpr int kFuThreads = 512;
constexpr int kFuQ = 64;          // per-warp word queue (8 warps share the block)
using FuShared = WcSharedT<kFuThreads / 32, kFuQ>;
constexpr size_t kFuSmemForce = 120 * 1024;   // dynamic smem >= half an SM: one CTA per SM

struct FusedArgs {
  const uint8_t* data;        // device alias of the registered (mapped) data set
  uint64_t nbytes;
  const uint64_t* off;        // device alias of the mapped offsets, nullptr: fixed records
  uint64_t rec_size;
  const uint64_t* ub;         // unit record bounds (U + 1), device
  const uint64_t* uby;        // unit byte bounds (U + 1), device
  uint32_t U, UB, UR;         // units; bytes / records per unit (caps)
  uint32_t n_load;            // loader CTAs (blockIdx < n_load); the rest consume
  uint8_t* ring;              // R slots of slot_bytes: [UB + 32 text][UR x 8 offsets]
  uint32_t R, slot_bytes;
  unsigned long long* ready;  // R: unit + 1 whose bytes the slot holds (zeroed by the run)
  unsigned long long* done;   // R: unit + 1 the slot was last consumed for (zeroed by the run)
  WcEntry* table;
  uint64_t mask;
  unsigned long long* used;
  int* err;
  unsigned long long* prof;   // optional: [0] consumer wait ns, [1] consumer compute ns, [2] consumer ns,
                              //           [3] loader wait ns, [4] loader copy ns
  // DMA-fed mode (n_load == 0): the copy engine fills K batch slots (consecutive units), each followed
  // by a stream-ordered flag write (ready[slot] = batch + 1); consumers count a batch's units done
  // and the last one releases the slot (done[slot] = batch + 1) for the DMA of batch + K
  const uint32_t* ubatch;     // U: unit -> batch
  const uint64_t* bby;        // NB + 1: batch byte bounds
  const uint64_t* brec;       // NB + 1: batch record bounds
  const uint32_t* bunits;     // NB: units per batch
  uint32_t K;                 // batch slots
  uint64_t bslot_bytes;       // slot: [btext + 64 text][offsets]
  uint64_t btext;
  unsigned int* bcnt;         // K: units of the slot's batch consumed (zeroed by the run)
};

__device__ __forceinline__ unsigned long long gtime() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ unsigned long long ld_acquire(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release(unsigned long long* p, unsigned long long v) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
constexpr unsigned long long kSpinLimitNs = 2000000000ull;   // 2 s: a stuck pipeline reports, never hangs

__global__ void __launch_bounds__(kFuThreads, 1) k_wc_fused(FusedArgs a) {
  extern __shared__ __align__(128) unsigned char fu_smem[];
  __shared__ FuShared sh;
  __shared__ int s_abort;
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  if (tid == 0) s_abort = 0;
  __syncthreads();
  const unsigned long long t_start = gtime();
  if (blockIdx.x < a.n_load) {
    // ------------------------------------------------------------ loader: stages 1-3
    unsigned long long t_wait = 0;
    for (uint32_t u = blockIdx.x; u < a.U; u += a.n_load) {
      const uint32_t sl = u % a.R;
      const unsigned long long tw = gtime();
      if (tid == 0 && u >= a.R) {   // the slot's previous unit (u - R) must have been copied out
        while (ld_acquire(&a.done[sl]) < u - a.R + 1)
          if (gtime() - tw > kSpinLimitNs) { atomicOr(a.err, kErrFusedTimeout); s_abort = 1; break; }
      }
      __syncthreads();
      if (s_abort) break;
      t_wait += gtime() - tw;
      uint8_t* slot = a.ring + (size_t)sl * a.slot_bytes;
      const uint64_t lo = a.ub[u], hi = a.ub[u + 1];
      const uint64_t b0 = a.uby[u], b1 = a.uby[u + 1];
      if (a.off) {
        uint64_t* o = reinterpret_cast<uint64_t*>(slot + a.UB + 32);
        for (uint64_t j = tid; j < hi - lo; j += blockDim.x) o[j] = __ldcs(a.off + lo + j);
      }
      const uintptr_t first = ((uintptr_t)(a.data + b0)) & ~(uintptr_t)15;
      const uintptr_t last = ((uintptr_t)(a.data + b1) + 15) & ~(uintptr_t)15;
      const uintptr_t dlo = (uintptr_t)a.data, dhi = (uintptr_t)(a.data + a.nbytes);
      const uint32_t nw = (uint32_t)((last - first) >> 4);
      // 4 independent 16-B host loads per thread in flight, then their stores
      for (uint32_t k0 = tid; k0 < nw; k0 += 4 * blockDim.x) {
        uint4 v[4];
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          const uint32_t k = k0 + q * blockDim.x;
          const uintptr_t p = first + 16 * (uintptr_t)k;
          v[q] = make_uint4(0, 0, 0, 0);
          if (k < nw) {
            if (p >= dlo && p + 16 <= dhi) {
              v[q] = __ldcs(reinterpret_cast<const uint4*>(p));
            } else {   // a word straddling the data set's edge: only its in-range bytes are read
              uint32_t ww[4] = {0, 0, 0, 0};
              for (int z = 0; z < 16; ++z)
                if (p + z >= dlo && p + z < dhi) ww[z >> 2] |= (uint32_t)*reinterpret_cast<const uint8_t*>(p + z) << (8 * (z & 3));
              v[q] = make_uint4(ww[0], ww[1], ww[2], ww[3]);
            }
          }
        }
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          const uint32_t k = k0 + q * blockDim.x;
          if (k < nw) __stcg(reinterpret_cast<uint4*>(slot) + k, v[q]);
        }
      }
      __threadfence();
      __syncthreads();
      if (tid == 0) st_release(&a.ready[sl], (unsigned long long)u + 1);
    }
    if (a.prof && tid == 0) {
      atomicAdd(&a.prof[3], t_wait);
      atomicAdd(&a.prof[4], gtime() - t_start - t_wait);
    }
    return;
  }
  // -------------------------------------------------------------- consumer: stage 4
  const uint32_t nc = gridDim.x - a.n_load, ci = blockIdx.x - a.n_load;
  const unsigned lt = (1u << lane) - 1;
  for (int i = tid; i < kWcTab; i += blockDim.x) { sh.k1[i] = 0; sh.k2[i] = 0; sh.cnt[i] = 0; }
  uint8_t* txt_s = fu_smem;                                                   // UB + 64 bytes
  uint64_t* offs = reinterpret_cast<uint64_t*>(fu_smem + a.UB + 64);          // UR entries
  uint32_t* Dm = reinterpret_cast<uint32_t*>(offs + a.UR);                     // (UB + 64) / 32 + 2 entries
  uint32_t* Bm = Dm + (a.UB + 64) / 32 + 2;
  unsigned long long t_wait = 0, t_comp = 0;
  const bool dma = a.n_load == 0;
  for (uint32_t u = ci; u < a.U; u += nc) {
    const uint32_t b = dma ? a.ubatch[u] : u;      // what the flag names: the unit, or its batch
    const uint32_t sl = dma ? b % a.K : u % a.R;
    const unsigned long long tw = gtime();
    if (tid == 0) {
      while (ld_acquire(&a.ready[sl]) != (unsigned long long)b + 1)
        if (gtime() - tw > kSpinLimitNs) { atomicOr(a.err, kErrFusedTimeout); s_abort = 1; break; }
    }
    __syncthreads();
    if (s_abort) break;
    const unsigned long long t1 = gtime();
    t_wait += t1 - tw;
    const uint64_t lo = a.ub[u], hi = a.ub[u + 1];
    const uint64_t base = a.uby[u];
    const uint32_t nrec = (uint32_t)(hi - lo), A = (uint32_t)(a.uby[u + 1] - base);
    {   // slot -> shared memory (L2 reads: the flag's acquire orders them; .cg bypasses stale L1 lines)
      const uint32_t sh0 = (uint32_t)(((uintptr_t)(a.data + base)) & 15);
      const uint32_t nw = (sh0 + A + 15) >> 4;
      const uint4* src;
      const uint64_t* so;
      if (dma) {   // the unit inside its batch: the batch's byte 0 sits at (data + bby[b]) mod 16
        const uint8_t* bs = a.ring + (size_t)sl * a.bslot_bytes;
        const uint64_t q = (((uintptr_t)(a.data + a.bby[b])) & 15) + (base - a.bby[b]);
        src = reinterpret_cast<const uint4*>(bs + (q & ~15ull));
        so = reinterpret_cast<const uint64_t*>(bs + a.btext + 64) + (lo - a.brec[b]);
      } else {
        const uint8_t* slot = a.ring + (size_t)sl * a.slot_bytes;
        src = reinterpret_cast<const uint4*>(slot);
        so = reinterpret_cast<const uint64_t*>(slot + a.UB + 32);
      }
      for (uint32_t k = tid; k < nw; k += blockDim.x) reinterpret_cast<uint4*>(txt_s)[k] = __ldcg(src + k);
      if (a.off)
        for (uint32_t j = tid; j < nrec; j += blockDim.x) offs[j] = __ldcg(so + j);
    }
    __syncthreads();
    if (tid == 0) {
      if (!dma) {
        st_release(&a.done[sl], (unsigned long long)u + 1);   // slot free for unit u + R
      } else if (atomicAdd(&a.bcnt[sl], 1u) + 1 == a.bunits[b]) {
        a.bcnt[sl] = 0;                                       // last unit of the batch out of the slot:
        st_release(&a.done[sl], (unsigned long long)b + 1);  // the DMA of batch b + K may refill it
      }
    }
    // ---- stage 1 (record boundaries -> break bits) + stage 4, word-parallel. Positions q are
    // relative to the 16-B-aligned copy (the unit's byte 0 at q = sh0). Two bitmaps over the unit:
    //   Dm: byte q is a delimiter (or outside the unit), Bm: a record starts at q (a word break, A10/A19);
    // a word starts at q iff q is not a delimiter and q-1 is one or q starts a record, and ends at
    // the next delimiter or record start. Each thread owns the words starting in its 32-byte segments,
    // so the per-byte work is one SWAR classification and the hash of the word's bytes.
    const uint32_t sh0 = (uint32_t)(((uintptr_t)(a.data + base)) & 15);
    const uint32_t qend = sh0 + A;                       // first position past the unit
    const uint32_t nseg = (qend + 31) >> 5;
    for (uint32_t i = tid; i <= nseg; i += blockDim.x) Bm[i] = 0;
    __syncthreads();
    for (uint32_t j = 1 + tid; j < nrec; j += blockDim.x) {   // record starts after the unit's first
      const uint32_t q = sh0 + (a.off ? (uint32_t)(offs[j] - base) : (uint32_t)((lo + j) * a.rec_size - base));
      atomicOr(&Bm[q >> 5], 1u << (q & 31));
    }
    for (uint32_t i = tid; i <= nseg; i += blockDim.x) {
      uint32_t dm = 0xffffffffu;
      if (i < nseg) {
        dm = 0;
        const uint32_t* wp = reinterpret_cast<const uint32_t*>(txt_s) + 8 * i;
#pragma unroll
        for (int k = 0; k < 8; ++k) {
          const uint32_t x = wp[k];
          // per byte 0xff where x == ' ' or 9 <= x <= 13, gathered to 4 bits
          const uint32_t f = (__vcmpeq4(x, 0x20202020u) | (__vcmpgeu4(x, 0x09090909u) & __vcmpleu4(x, 0x0d0d0d0du)))
                             & 0x01010101u;
          dm |= ((f * 0x01020408u) >> 24) << (4 * k);
        }
        const uint32_t q0 = 32 * i;   // positions outside [sh0, qend) count as delimiters
        if (q0 < sh0) dm |= sh0 - q0 >= 32 ? 0xffffffffu : (1u << (sh0 - q0)) - 1;
        if (q0 + 32 > qend) dm |= qend <= q0 ? 0xffffffffu : ~((1u << (qend - q0)) - 1);
      }
      Dm[i] = dm;
    }
    __syncthreads();
    const uint8_t* tb = txt_s;
    int qn = 0;   // warp-uniform queue fill
    for (uint32_t i0 = 0; i0 < nseg; i0 += blockDim.x) {
      const uint32_t i = i0 + tid;
      uint32_t S = 0;
      if (i < nseg) {
        const uint32_t dm = Dm[i], bm = Bm[i];
        const uint32_t prevd = i ? (Dm[i - 1] >> 31) : 1u;
        S = ~dm & ((dm << 1) | prevd | bm);
      }
      // one word per lane per round: hash it, then the warp appends the round's words to its queue
      while (__any_sync(kFull, S != 0)) {
        const bool has = S != 0;
        uint64_t h1 = 0, h2 = 0;
        uint32_t q = 0, len = 0;
        if (has) {
          const uint32_t bit = __ffs(S) - 1;
          S &= S - 1;
          q = 32 * i + bit;
          // end: the next break bit (delimiter or record start) after q
          uint32_t seg = i;
          uint32_t m = (Dm[seg] | Bm[seg]) & (bit == 31 ? 0u : ~((2u << bit) - 1));
          while (!m) {
            ++seg;
            m = Dm[seg] | Bm[seg];   // Dm[nseg] is all ones: a word always ends
          }
          const uint32_t r = 32 * seg + __ffs(m) - 1;
          len = r - q;
          h1 = 0xcbf29ce484222325ull;
          h2 = 0x84222325cbf29ce4ull;
          for (uint32_t x = q; x < r; ++x) {
            const uint32_t ch = tb[x];
            h1 = (h1 ^ ch) * 0x100000001b3ull;
            h2 = (h2 + ch + 1) * 0x9E3779B97F4A7C15ull;
            h2 ^= h2 >> 29;
          }
        }
        const unsigned m = __ballot_sync(kFull, has);
        if (has) {
          const uint64_t occ = base + (q - sh0);
          if (len >= (1u << 24) || occ >= (1ull << 40)) atomicOr(a.err, kErrWordTooLong);
          const int k = qn + __popc(m & lt);
          sh.qk1[w][k] = h1;
          sh.qk2[w][k] = h2;
          sh.qol[w][k] = (occ << 24) | len;
        }
        qn += __popc(m);
        if (qn > kFuQ - 32) {
          wc_flush_queue(sh, w, lane, qn, a.table, a.mask, a.used, a.err);
          qn = 0;
        }
      }
    }
    if (qn) wc_flush_queue(sh, w, lane, qn, a.table, a.mask, a.used, a.err);
    // the block table caches this unit's hot words; empty it into the global table before the next
    // unit (a table kept across units would fill with early words and send the hot ones global)
    __syncthreads();
    wc_flush_block<FuShared, kWcTab / kFuThreads>(sh, tid, kFuThreads, a.table, a.mask, a.used, a.err, true);
    __syncthreads();
    t_comp += gtime() - t1;
  }
  if (a.prof && tid == 0) {
    atomicAdd(&a.prof[0], t_wait);
    atomicAdd(&a.prof[1], t_comp);
    atomicAdd(&a.prof[2], gtime() - t_start);
  }
}

// ------------------------------------------------------------------------------------------
// C2 grep (MCA analogue): key = first strnlen(32) bytes of the record's 32-byte key
// field (staged as words 2j, 2j+1 of the lane); match iff the pattern is a substring. Output
// indices are ascending. Chunks compute in any order (per-slot streams). Per chunk:
//   k_grep_count  each warp streams its tiles through shared memory (WarpTileStream) and writes
//                 per-lane match masks (bit j = record j of the lane) and per-tile match counts;
//   k_grep_scan   one block: the chunk's match count, its run [base, base+n) of a match pool
//                 (one atomicAdd), and each tile's output base;
//   k_grep_write  one warp per tile turns the masks into ascending record indices (no key re-read).
// After the last chunk one pass copies the runs into chunk order (k_grep_order).

struct Key32 { uint32_t w[8]; };   // the key field, little-endian words

// bit x set iff key byte x == the byte replicated in `rep` (SWAR compare of 4 bytes per word; the
// 0/1 byte flags at bits 0, 8, 16, 24 are gathered to bits 24..27 by one multiply)
__device__ __forceinline__ uint32_t eqmask32(const Key32& k, uint32_t rep) {
  uint32_t m = 0;
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const uint32_t t = __vcmpeq4(k.w[i], rep) & 0x01010101u;
    m |= ((t * 0x01020408u) >> 24) << (4 * i);
  }
  return m;
}

// Match bits of every start position: bit x set iff x + plen <= kl and key[x + i] == pat[i] for
// all i < plen, i.e. AND_i (eqmask(pat[i]) >> i) restricted to the positions that fit in the key.
__device__ __forceinline__ bool grep_match(const Key32& k, const GrepParams& p) {
  if (p.plen == 0) return true;
  const uint32_t z = eqmask32(k, 0u);
  const int kl = z ? __ffs((int)z) - 1 : 32;   // strnlen(key, 32)
  const int plen = (int)p.plen;
  if (kl < plen) return false;
  const int fit = kl - plen + 1;               // start positions 0 .. kl - plen
  uint32_t M = fit >= 32 ? 0xffffffffu : ((1u << fit) - 1);
#pragma unroll
  for (int i = 0; i < 32; ++i) {   // unrolled: pattern bytes come from the constant bank, not a stack copy
    if (i >= plen || !M) break;
    M &= eqmask32(k, (uint32_t)p.pat[i] * 0x01010101u) >> i;
  }
  return M != 0;
}

__device__ __forceinline__ Key32 key_at(const uint8_t* row0, int lane) {  // rows 2j, 2j+1 (smem or HBM)
  const uint4 a = *reinterpret_cast<const uint4*>(row0 + lane * 16);
  const uint4 b = *reinterpret_cast<const uint4*>(row0 + 512 + lane * 16);
  return Key32{{a.x, a.y, a.z, a.w, b.x, b.y, b.z, b.w}};
}

constexpr int kGrepThreads = 256;
constexpr uint32_t kGrepRows = 8;    // rows per piece: 4 keys of 2 words

template <bool kTma>
__global__ void __launch_bounds__(kGrepThreads) k_grep_count(Chunk c, const uint8_t* __restrict__ stage,
                                                             const LaneDesc* __restrict__ lanes,
                                                             const uint64_t* __restrict__ tile_base, GrepParams p,
                                                             uint32_t* __restrict__ tilecnt,
                                                             uint32_t* __restrict__ lanemask) {
  extern __shared__ __align__(128) unsigned char smem_raw[];
  constexpr uint32_t nwarp = kGrepThreads / 32;
  const uint32_t wid = threadIdx.x >> 5, lane = threadIdx.x & 31;
  WarpTileStream<kTma> ts = warp_stream<kTma>(smem_raw, nwarp, kGrepRows, stage, tile_base, c.ntiles);
  ts.begin(blockIdx.x * nwarp + wid);
  uint32_t mask = 0, cnt = 0;
  while (ts.valid()) {
    const uint32_t nrec = lanes[(size_t)ts.w * 32 + lane].nrec;
    if (ts.p == 0) mask = cnt = 0;
    uint32_t nw, np, nK;
    const uint8_t* piece = ts.acquire(nw, np, nK);
    const uint32_t r0 = ts.p * kGrepRows;
    const uint32_t j1 = min(min(ts.K, r0 + kGrepRows) / 2, nrec);
    for (uint32_t j = r0 / 2; j < j1; ++j) {
      const uint32_t m = grep_match(key_at(piece + (size_t)(2 * j - r0) * 512, lane), p);
      cnt += m;
      if (j < 32) mask |= m << j;
    }
    if ((ts.p + 1) * kGrepRows >= ts.K) {   // last piece of the tile
      lanemask[(size_t)ts.w * 32 + lane] = mask;
      const uint32_t tot = __reduce_add_sync(kFull, cnt);
      if (lane == 0) tilecnt[ts.w] = tot;
    }
    ts.release(nw, np, nK);
  }
}

// tiles with no staged rows were never visited by k_grep_count: they count zero
__global__ void __launch_bounds__(1024) k_grep_scan(const uint32_t* __restrict__ tilecnt,
                                                    const uint64_t* __restrict__ tile_base, uint32_t ntiles,
                                                    unsigned long long* cursor, unsigned long long* tilebase_out,
                                                    unsigned long long* chunk_run) {
  __shared__ unsigned long long warp_sums[32];
  __shared__ unsigned long long carry;
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  auto count = [&](uint32_t i) -> unsigned long long {
    return i < ntiles && tile_base[i + 1] > tile_base[i] ? tilecnt[i] : 0ull;
  };
  // the chunk's match count, then its run in the pool: [base, base + total)
  unsigned long long part = 0;
  for (uint32_t i = threadIdx.x; i < ntiles; i += 1024) part += count(i);
#pragma unroll
  for (int o = 16; o; o >>= 1) part += __shfl_xor_sync(kFull, part, o);
  if (lane == 0) warp_sums[wid] = part;
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long tot = 0;
    for (int w = 0; w < 32; ++w) tot += warp_sums[w];
    carry = atomicAdd(cursor, tot);
    chunk_run[0] = carry;
    chunk_run[1] = tot;
  }
  __syncthreads();
  for (uint32_t base = 0; base < ntiles; base += 1024) {
    const uint32_t i = base + threadIdx.x;
    const unsigned long long v = count(i);
    unsigned long long x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const unsigned long long y = __shfl_up_sync(kFull, x, o);
      if (lane >= o) x += y;
    }
    if (lane == 31) warp_sums[wid] = x;
    __syncthreads();
    if (wid == 0) {
      unsigned long long s = warp_sums[lane];
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const unsigned long long y = __shfl_up_sync(kFull, s, o);
        if (lane >= o) s += y;
      }
      warp_sums[lane] = s;
    }
    __syncthreads();
    const unsigned long long excl = carry + (wid ? warp_sums[wid - 1] : 0) + x - v;
    if (i < ntiles) tilebase_out[i] = excl;
    __syncthreads();
    if (threadIdx.x == 1023) carry = excl + v;
    __syncthreads();
  }
}

// Block c copies chunk c's run of the pool to its place in chunk order (the sum of the runs of
// chunks 0..c-1), clipped to cap (overflow was already flagged by k_grep_write).
__global__ void __launch_bounds__(256) k_grep_order(const unsigned long long* __restrict__ runs, uint32_t C,
                                                    const uint64_t* __restrict__ pool, uint64_t* __restrict__ out,
                                                    uint64_t cap) {
  __shared__ unsigned long long sh[8];
  __shared__ unsigned long long s_dst;
  const uint32_t c = blockIdx.x;
  unsigned long long before = 0;
  for (uint32_t i = threadIdx.x; i < c; i += blockDim.x) before += runs[2 * i + 1];
#pragma unroll
  for (int o = 16; o; o >>= 1) before += __shfl_down_sync(kFull, before, o);
  if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = before;
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long t = 0;
    for (int w = 0; w < (int)(blockDim.x >> 5); ++w) t += sh[w];
    s_dst = t;
  }
  __syncthreads();
  const unsigned long long dst = s_dst, src = runs[2 * c], n = runs[2 * c + 1];
  for (unsigned long long k = threadIdx.x; k < n; k += blockDim.x)
    if (dst + k < cap && src + k < cap) out[dst + k] = pool[src + k];
}

// One warp per tile: lane t's matches go to tilebase_out[w] + (matches of lanes before t), in
// record order. Lanes of more than 32 records (a lane_bytes override) re-test their keys from HBM.
__global__ void __launch_bounds__(256) k_grep_write(Chunk c, const uint8_t* __restrict__ stage,
                                                    const LaneDesc* __restrict__ lanes,
                                                    const uint64_t* __restrict__ tile_base, GrepParams p,
                                                    const unsigned long long* __restrict__ tilebase_out,
                                                    const uint32_t* __restrict__ lanemask,
                                                    uint64_t* __restrict__ out, int* err) {
  const uint32_t w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (w >= c.ntiles || tile_base[w + 1] == tile_base[w]) return;   // whole warps leave together
  const LaneDesc d = lanes[(size_t)w * 32 + lane];
  const uint8_t* tile = stage + tile_base[w];
  uint32_t mask = 0, cnt = 0;
  if (d.nrec <= 32) {
    mask = d.nrec ? lanemask[(size_t)w * 32 + lane] : 0;
    cnt = __popc(mask);
  } else {
    for (uint32_t j = 0; j < d.nrec; ++j) cnt += grep_match(key_at(tile + (size_t)2 * j * 512, lane), p);
  }
  uint32_t x = cnt;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(kFull, x, o);
    if (lane >= o) x += y;
  }
  unsigned long long pos = tilebase_out[w] + x - cnt;
  auto emit = [&](uint32_t j) {
    if (pos < p.cap) out[pos] = p.first_index + d.first + j;
    else atomicOr(err, kErrOutOverflow);
    ++pos;
  };
  if (d.nrec <= 32) {
    for (; mask; mask &= mask - 1) emit((uint32_t)__ffs((int)mask) - 1);
  } else if (cnt) {
    for (uint32_t j = 0; j < d.nrec; ++j)
      if (grep_match(key_at(tile + (size_t)2 * j * 512, lane), p)) emit(j);
  }
}

// ------------------------------------------------------------------------------------------
// C5 group-by: records {u32 key, u32 qty, f64 amount} staged one word per record.
// Each warp streams its tiles through shared memory with bulk copies (WarpTileStream, tma.cuh:
// the copy of the next piece is in flight while the warp aggregates the current one) into a
// block-private shared-memory table (count, qty, amount), flushed once per block.

constexpr int kGbThreads = 512;

__host__ __device__ constexpr uint32_t groupby_rows(uint32_t G) { return G <= 4096 ? 8 : 4; }

template <bool kTma>
__global__ void __launch_bounds__(kGbThreads) k_groupby(Chunk c, const uint8_t* __restrict__ stage,
                                                        const LaneDesc* __restrict__ lanes,
                                                        const uint64_t* __restrict__ tile_base, uint32_t G,
                                                        unsigned long long* gcount, unsigned long long* gqty,
                                                        double* gamount, int* err) {
  extern __shared__ __align__(128) unsigned char smem_raw[];
  constexpr uint32_t nwarp = kGbThreads / 32;
  const uint32_t rows = groupby_rows(G);
  const uint32_t wid = threadIdx.x >> 5, lane = threadIdx.x & 31;
  WarpTileStream<kTma> ts = warp_stream<kTma>(smem_raw, nwarp, rows, stage, tile_base, c.ntiles);
  double* s_amt = reinterpret_cast<double*>(smem_raw + stream_smem<kTma>(nwarp, rows));
  unsigned int* s_cnt = reinterpret_cast<unsigned int*>(s_amt + G);
  unsigned int* s_qty = s_cnt + G;
  for (uint32_t g = threadIdx.x; g < G; g += blockDim.x) { s_amt[g] = 0.0; s_cnt[g] = 0; s_qty[g] = 0; }
  __syncthreads();
  ts.begin(blockIdx.x * nwarp + wid);
  while (ts.valid()) {
    const uint32_t nrec = lanes[(size_t)ts.w * 32 + lane].nrec;
    uint32_t nw, np, nK;
    const uint8_t* piece = ts.acquire(nw, np, nK);
    const uint32_t r0 = ts.p * rows;
    const uint32_t r1 = min(min(ts.K, r0 + rows), nrec);
    for (uint32_t r = r0; r < r1; ++r) {
      const uint4 v = *reinterpret_cast<const uint4*>(piece + (size_t)(r - r0) * 512 + lane * 16);
      const uint32_t key = v.x;
      if (key >= G) { atomicOr(err, kErrKeyRange); continue; }
      const double amt = __hiloint2double((int)v.w, (int)v.z);
      atomicAdd(&s_cnt[key], 1u);
      atomicAdd(&s_qty[key], v.y);
      atomicAdd(&s_amt[key], amt);
    }
    ts.release(nw, np, nK);
  }
  __syncthreads();
  for (uint32_t g = threadIdx.x; g < G; g += blockDim.x) {
    if (s_cnt[g]) {
      atomicAdd(&gcount[g], (unsigned long long)s_cnt[g]);
      atomicAdd(&gqty[g], (unsigned long long)s_qty[g]);
      atomicAdd(&gamount[g], s_amt[g]);
    }
  }
}

// ------------------------------------------------------------------------------------------
// C3 k-means step (P:289-305 clusterKernel/findClosestCluster): fp32 distance in the exact
// order of DESIGN.md reading A13 (__fsub_rn, __fmaf_rn, j ascending), argmin with ties to the
// lowest k; per-block shared sums (fp64) and counts, flushed once per block.

// Each warp streams its tiles through shared memory (WarpTileStream, 2 points per piece) and
// evaluates four centroids at a time: four independent fmaf chains, each in the order of A13,
// compared in ascending k afterwards, so the argmin (ties to the lowest k) is bit-identical to
// the one-centroid-at-a-time loop while the FMA pipes see four chains to interleave.
constexpr int kKmThreads = 512;
constexpr uint32_t kKmRows = 8;   // rows per piece: 2 points of 4 words

// Exact fp32 -> fp64 widening with integer ops for normal numbers and zeros (rebias the exponent,
// shift the mantissa); subnormals, infinities and NaNs take the conversion instruction. ncu showed
// the 16 conversions per point saturating the XU pipe (122% of its sustained rate) in k_kmeans.
__device__ __forceinline__ double widen(float f) {
  const uint32_t u = __float_as_uint(f);
  const uint32_t e = (u >> 23) & 0xffu;
  const uint64_t sign = (uint64_t)(u >> 31) << 63;
  if (e - 1u < 0xfeu)
    return __longlong_as_double((long long)(sign | ((uint64_t)(e + 896u) << 52) | ((uint64_t)(u & 0x7fffffu) << 29)));
  if ((u << 1) == 0) return __longlong_as_double((long long)sign);
  return (double)f;
}

__device__ __forceinline__ float km_dist(const float* x, const float* m) {
  float acc = 0.0f;
#pragma unroll
  for (int q = 0; q < 16; ++q) {
    const float df = __fsub_rn(x[q], m[q]);
    acc = __fmaf_rn(df, df, acc);
  }
  return acc;
}

template <bool kTma>
__global__ void __launch_bounds__(kKmThreads) k_kmeans(Chunk c, const uint8_t* __restrict__ stage,
                                                       const LaneDesc* __restrict__ lanes,
                                                       const uint64_t* __restrict__ tile_base,
                                                       const float* __restrict__ mu, uint32_t K, uint64_t first_index,
                                                       unsigned long long* gcount, double* gsum,
                                                       unsigned long long* gchk, int32_t* __restrict__ cid_out) {
  extern __shared__ __align__(128) unsigned char smem_raw[];
  constexpr uint32_t nwarp = kKmThreads / 32;
  const uint32_t wid = threadIdx.x >> 5, lane = threadIdx.x & 31;
  WarpTileStream<kTma> ts = warp_stream<kTma>(smem_raw, nwarp, kKmRows, stage, tile_base, c.ntiles);
  double* s_sum = reinterpret_cast<double*>(smem_raw + stream_smem<kTma>(nwarp, kKmRows));   // K*16
  float* s_mu = reinterpret_cast<float*>(s_sum + (size_t)K * 16);                             // K*16
  unsigned int* s_cnt = reinterpret_cast<unsigned int*>(s_mu + (size_t)K * 16);
  for (uint32_t i = threadIdx.x; i < K * 16; i += blockDim.x) { s_sum[i] = 0.0; s_mu[i] = mu[i]; }
  for (uint32_t i = threadIdx.x; i < K; i += blockDim.x) s_cnt[i] = 0;
  __syncthreads();
  unsigned long long chk = 0;
  ts.begin(blockIdx.x * nwarp + wid);
  while (ts.valid()) {
    const LaneDesc d = lanes[(size_t)ts.w * 32 + lane];
    uint32_t nw, np, nK;
    const uint8_t* piece = ts.acquire(nw, np, nK);
    const uint32_t r0 = ts.p * kKmRows;
    const uint32_t j1 = min(min(ts.K, r0 + kKmRows) / 4, d.nrec);
    const uint32_t jw = __reduce_max_sync(kFull, j1);   // warp-uniform trip count (lanes past j1 idle)
    for (uint32_t j = r0 / 4; j < jw; ++j) {
      const bool valid = j < j1;
      float x[16];
#pragma unroll
      for (int w = 0; w < 4; ++w) {
        const uint4 v = *reinterpret_cast<const uint4*>(piece + (size_t)(4 * j + w - r0) * 512 + lane * 16);
        x[4 * w + 0] = __uint_as_float(v.x);
        x[4 * w + 1] = __uint_as_float(v.y);
        x[4 * w + 2] = __uint_as_float(v.z);
        x[4 * w + 3] = __uint_as_float(v.w);
      }
      uint32_t best = 0;
      float bestd = 0.0f;
      uint32_t k = 0;
      for (; k + 4 <= K; k += 4) {
        const float a0 = km_dist(x, s_mu + (k + 0) * 16);
        const float a1 = km_dist(x, s_mu + (k + 1) * 16);
        const float a2 = km_dist(x, s_mu + (k + 2) * 16);
        const float a3 = km_dist(x, s_mu + (k + 3) * 16);
        if (k == 0 || a0 < bestd) { bestd = a0; best = k; }
        if (a1 < bestd) { bestd = a1; best = k + 1; }
        if (a2 < bestd) { bestd = a2; best = k + 2; }
        if (a3 < bestd) { bestd = a3; best = k + 3; }
      }
      for (; k < K; ++k) {
        const float a0 = km_dist(x, s_mu + k * 16);
        if (k == 0 || a0 < bestd) { bestd = a0; best = k; }
      }
      // warp aggregation by cluster: lanes that chose the same centroid form a group; its leader pulls
      // the members' coordinates (one fp32 shuffle each, summed exactly in fp64) and makes the group's
      // 16 shared fp64 adds — no intra-warp contention on one cluster's sums, fewer CAS loops
      const unsigned vmask = __ballot_sync(kFull, valid);
      const unsigned grp = __match_any_sync(kFull, valid ? best : 0xffffffffu) & vmask;
      const bool leader = valid && lane == __ffs(grp) - 1;
      unsigned others = leader ? grp & ~(1u << lane) : 0u;
      double acc[16];
#pragma unroll
      for (int q = 0; q < 16; ++q) acc[q] = widen(x[q]);
      while (__any_sync(kFull, others != 0)) {
        const int src = others ? __ffs(others) - 1 : (int)lane;
        others &= others - 1;
#pragma unroll
        for (int q = 0; q < 16; ++q) {
          const float y = __shfl_sync(kFull, x[q], src);
          if (src != (int)lane) acc[q] += widen(y);
        }
      }
      if (leader) {
        atomicAdd(&s_cnt[best], (unsigned)__popc(grp));
#pragma unroll
        for (int q = 0; q < 16; ++q) atomicAdd(&s_sum[best * 16 + q], acc[q]);
      }
      if (valid) {
        chk += mix64(((first_index + d.first + j) << 8) ^ (uint64_t)best);
        if (cid_out) cid_out[d.first + j - c.lo] = (int32_t)best;
      }
    }
    ts.release(nw, np, nK);
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) chk += __shfl_xor_sync(kFull, chk, o);  // wraps mod 2^64
  __syncthreads();
  for (uint32_t i = threadIdx.x; i < K * 16; i += blockDim.x)
    if (s_sum[i] != 0.0) atomicAdd(&gsum[i], s_sum[i]);
  for (uint32_t i = threadIdx.x; i < K; i += blockDim.x)
    if (s_cnt[i]) atomicAdd(&gcount[i], (unsigned long long)s_cnt[i]);
  if (lane == 0) atomicAdd(gchk, chk);
}

}  // namespace

void launch_wc(const Chunk& c, const uint8_t* stage, const LaneDesc* lanes, const uint64_t* tile_base,
               const uint64_t* meta, uint64_t rec_size, WcEntry* table, uint64_t mask, unsigned long long* used,
               int* err, cudaStream_t s) {
  constexpr int kSub = 8;  // sub-threads per 256-B lane (sweep: 2/4/8/16, profiles/r01_wc_sweep.md)
  const uint32_t grid = (c.L * kSub + kWcBlock - 1) / kWcBlock;
  k_wc<kSub><<<grid, kWcBlock, 0, s>>>(c, stage, lanes, tile_base, meta, rec_size, table, mask, used, err);
}

uint32_t wc_fused_slot_bytes(uint32_t UB, uint32_t UR) { return (UB + 32 + UR * 8 + 255) / 256 * 256; }

size_t wc_fused_smem(uint32_t UB, uint32_t UR) {
  return std::max<size_t>(kFuSmemForce, (size_t)UB + 64 + (size_t)UR * 8 + 2 * ((size_t)(UB + 64) / 32 + 2) * 4);
}

int wc_fused_grid() { return device_sms(); }

cudaError_t launch_wc_fused(const uint8_t* data, uint64_t nbytes, const uint64_t* off, uint64_t rec_size,
                            const uint64_t* ub, const uint64_t* uby, uint32_t U, uint32_t UB, uint32_t UR, int grid,
                            uint32_t n_load, uint8_t* ring, uint32_t R, unsigned long long* ready,
                            unsigned long long* done, WcEntry* table, uint64_t mask, unsigned long long* used,
                            int* err, unsigned long long* prof, const FusedDma* dma, cudaStream_t s) {
  FusedArgs a{data, nbytes, off, rec_size, ub, uby, U, UB, UR, n_load, ring, R, wc_fused_slot_bytes(UB, UR),
              ready, done, table, mask, used, err, prof};
  if (dma) {
    a.n_load = 0;
    a.ubatch = dma->ubatch;
    a.bby = dma->bby;
    a.brec = dma->brec;
    a.bunits = dma->bunits;
    a.K = dma->K;
    a.bslot_bytes = dma->bslot_bytes;
    a.btext = dma->btext;
    a.bcnt = dma->bcnt;
  }
  // cooperative: every CTA is co-resident (loaders and consumers wait on each other)
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(kFuThreads);
  cfg.dynamicSmemBytes = wc_fused_smem(UB, UR);
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeCooperative;
  at[0].val.cooperative = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, k_wc_fused, a);
}

uint32_t wc_fused_threads() { return kFuThreads; }

void launch_dbuf_wc(const uint8_t* raw, const uint64_t* meta, uint64_t lo, uint64_t hi, uint64_t base_byte,
                    uint64_t end_byte, uint64_t rec_size, WcEntry* table, uint64_t mask, unsigned long long* used,
                    int* err, cudaStream_t s) {
  k_dbuf_wc<<<device_sms() * 4, 256, 0, s>>>(raw, meta, lo, hi, base_byte, end_byte, rec_size, table, mask, used, err);
}

void launch_wc_compact(WcEntry* table, uint64_t slots, unsigned long long* n_out, unsigned long long* total,
                       uint64_t* off, uint32_t* len, uint64_t* cnt, uint64_t* h1, uint64_t* h2, uint64_t cap,
                       cudaStream_t s) {
  k_wc_compact<<<(unsigned)((slots + kCmpSlots - 1) / kCmpSlots), kCmpThreads, 0, s>>>(table, slots, n_out, total, off,
                                                                                     len, cnt, h1, h2, cap);
}

size_t grep_count_smem() { return stream_smem<true>(kGrepThreads / 32, kGrepRows); }

// Stage 4 reads the tiles through TMA bulk copies (persistent warps, double-buffered pieces) unless
// zero-copy gathers share the chunk's run (`tma` false): then plain loads, one tile per warp.
void launch_grep(const Chunk& c, const uint8_t* stage, const LaneDesc* lanes, const uint64_t* tile_base,
                 const GrepParams& p, uint32_t* tilecnt, uint32_t* lanemask, unsigned long long* cursor,
                 unsigned long long* tilebase_out, unsigned long long* chunk_run, uint64_t* out_idx, int* err,
                 int grid, bool tma, cudaStream_t s) {
  const uint32_t nwarp = kGrepThreads / 32;
  const uint32_t tile_blocks = std::max<uint32_t>(1, (c.ntiles + nwarp - 1) / nwarp);
  if (tma)
    k_grep_count<true><<<std::min<int>(grid, (int)tile_blocks), kGrepThreads, grep_count_smem(), s>>>(
        c, stage, lanes, tile_base, p, tilecnt, lanemask);
  else
    k_grep_count<false><<<tile_blocks, kGrepThreads, 0, s>>>(c, stage, lanes, tile_base, p, tilecnt, lanemask);
  k_grep_scan<<<1, 1024, 0, s>>>(tilecnt, tile_base, c.ntiles, cursor, tilebase_out, chunk_run);
  k_grep_write<<<tile_blocks, 256, 0, s>>>(c, stage, lanes, tile_base, p, tilebase_out, lanemask, out_idx, err);
}

void launch_grep_order(const unsigned long long* runs, uint32_t C, const uint64_t* pool, uint64_t* out, uint64_t cap,
                       cudaStream_t s) {
  if (C) k_grep_order<<<C, 256, 0, s>>>(runs, C, pool, out, cap);
}

size_t groupby_smem(uint32_t G, bool tma) {
  return (tma ? stream_smem<true>(kGbThreads / 32, groupby_rows(G)) : 0) + (size_t)G * 16;
}

void launch_groupby(const Chunk& c, const uint8_t* stage, const LaneDesc* lanes, const uint64_t* tile_base,
                    uint32_t G, unsigned long long* count, unsigned long long* qty, double* amount, int* err,
                    int grid, bool tma, cudaStream_t s) {
  // TMA: one 16-warp block per SM (stream buffers + table ~192 KB); plain loads: up to 3 per SM
  grid = std::min<int>(grid, (int)std::max<uint32_t>(1, (c.ntiles + kGbThreads / 32 - 1) / (kGbThreads / 32)));
  if (tma)
    k_groupby<true><<<grid, kGbThreads, groupby_smem(G, true), s>>>(c, stage, lanes, tile_base, G, count, qty, amount,
                                                                     err);
  else
    k_groupby<false><<<grid, kGbThreads, groupby_smem(G, false), s>>>(c, stage, lanes, tile_base, G, count, qty,
                                                                       amount, err);
}

size_t kmeans_smem(uint32_t K, bool tma) {
  return (tma ? stream_smem<true>(kKmThreads / 32, kKmRows) : 0) + (size_t)K * 16 * 8 + (size_t)K * 16 * 4 +
         (size_t)K * 4;
}

void launch_kmeans(const Chunk& c, const uint8_t* stage, const LaneDesc* lanes, const uint64_t* tile_base,
                   const float* mu, uint32_t K, uint64_t first_index, unsigned long long* count, double* sum,
                   unsigned long long* chk, int32_t* cid_out, int grid, bool tma, cudaStream_t s) {
  grid = std::min<int>(grid, (int)std::max<uint32_t>(1, (c.ntiles + kKmThreads / 32 - 1) / (kKmThreads / 32)));
  if (tma)
    k_kmeans<true><<<grid, kKmThreads, kmeans_smem(K, true), s>>>(c, stage, lanes, tile_base, mu, K, first_index,
                                                                   count, sum, chk, cid_out);
  else
    k_kmeans<false><<<grid, kKmThreads, kmeans_smem(K, false), s>>>(c, stage, lanes, tile_base, mu, K, first_index,
                                                                     count, sum, chk, cid_out);
}

cudaError_t configure_compute_kernels() {
  {   // the fused word count also holds its static FuShared tables: dynamic ring <= 227 KB - static
    const cudaError_t e = cudaFuncSetAttribute((const void*)k_wc_fused, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                               227 * 1024 - (int)sizeof(FuShared) - 2048);
    if (e != cudaSuccess) return e;
  }
  for (const void* f : {(const void*)k_groupby<true>, (const void*)k_groupby<false>, (const void*)k_kmeans<true>,
                        (const void*)k_kmeans<false>, (const void*)k_grep_count<true>}) {
    const cudaError_t e = cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, 220 * 1024);
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

}  // namespace bk
