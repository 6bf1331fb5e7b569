// kernels_compute.cu — pipeline stage 4 (Fig. 3):
// the compute kernels read their lane's words from the staged warp tiles (one coalesced
// 512-B access per warp per word, the point of the interleaved layout) and
// reduce with warp-level aggregation and block-level shared-memory tables before touching
// global memory (north_star: warp shuffles + block-level atomics).
#include "bk_internal.cuh"

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

struct WcShared {
  unsigned long long k1[kWcTab], k2[kWcTab], ol[kWcTab];
  unsigned int cnt[kWcTab];
  unsigned long long qk1[kWcBlock / 32][kWcQ], qk2[kWcBlock / 32][kWcQ], qol[kWcBlock / 32][kWcQ];
};

__device__ void tab_insert(WcShared& sh, WcEntry* table, uint64_t mask, unsigned long long k1,
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
__device__ __noinline__ void wc_flush_queue(WcShared& sh, int w, int lane, int n, WcEntry* table,
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
  constexpr int kPer = kWcTab / kWcBlock;
  unsigned long long k1[kPer], k2[kPer];
  ulonglong2 home[kPer];
#pragma unroll
  for (int m = 0; m < kPer; ++m) {
    const int i = threadIdx.x + m * kWcBlock;
    k1[m] = sh.k1[i];
    k2[m] = sh.k2[i];
    home[m] = k1[m] ? __ldcg(reinterpret_cast<const ulonglong2*>(&table[k1[m] & mask])) : make_ulonglong2(0, 0);
  }
#pragma unroll
  for (int m = 0; m < kPer; ++m) {
    const int i = threadIdx.x + m * kWcBlock;
    if (!k1[m]) continue;
    if (wc_home_hit(home[m], k1[m], k2[m])) atomicAdd(&table[k1[m] & mask].count, (unsigned long long)sh.cnt[i]);
    else wc_insert(table, mask, k1[m], k2[m], sh.ol[i], sh.cnt[i], used, err);
  }
}

__global__ void k_wc_compact(const WcEntry* __restrict__ table, uint64_t slots, unsigned long long* n_out,
                             uint64_t* off, uint32_t* len, uint64_t* cnt, uint64_t cap) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < slots; i += (uint64_t)gridDim.x * blockDim.x) {
    const WcEntry e = table[i];
    if (e.key1 == 0) continue;
    const unsigned long long p = atomicAdd(n_out, 1ull);
    if (p < cap) {
      off[p] = e.offlen >> 24;
      len[p] = (uint32_t)(e.offlen & 0xffffff);
      cnt[p] = e.count;
    }
  }
}

// ------------------------------------------------------------------------------------------
// C2 grep (MCA analogue): key = first strnlen(32) bytes of the record's 32-byte key
// field (staged as words 2j, 2j+1 of the lane); match iff the pattern is a substring. Output
// indices are ascending. Chunks compute in any order (per-slot streams): per chunk, block counts ->
// one-block scan that reserves the chunk's run in a match pool with one atomicAdd and records
// (pool offset, count) per chunk -> write; after the last chunk one pass copies the runs into
// chunk order (k_grep_order).

struct Key32 { uint64_t q[8]; };  // q[4..7] = 0: windows past byte 31 read zeros

__device__ __forceinline__ uint64_t window8(const Key32& k, int x) {  // bytes [x, x+8), x constant
  const int i = x >> 3, s = (x & 7) * 8;
  if (s == 0) return k.q[i];
  return (k.q[i] >> s) | (k.q[i + 1] << (64 - s));
}

__device__ __forceinline__ uint32_t strnlen32(const Key32& k) {
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const uint64_t v = k.q[i];
    const uint64_t z = (v - 0x0101010101010101ull) & ~v & 0x8080808080808080ull;  // first zero byte
    if (z) return 8 * i + (__ffsll((long long)z) - 1) / 8;
  }
  return 32;
}

__device__ __forceinline__ bool grep_match(const Key32& k, const GrepParams& p, const uint64_t* pw,
                                           const uint64_t* pm) {
  if (p.plen == 0) return true;
  const int kl = (int)strnlen32(k);
  const int plen = (int)p.plen;
  bool hit = false;
#pragma unroll
  for (int x = 0; x < 32; ++x) {
    bool ok = x + plen <= kl && (window8(k, x) & pm[0]) == pw[0];
    if (plen > 8) ok = ok && (window8(k, x + 8) & pm[1]) == pw[1];
    if (plen > 16) ok = ok && (window8(k, x + 16) & pm[2]) == pw[2];
    if (plen > 24) ok = ok && (window8(k, x + 24) & pm[3]) == pw[3];
    hit = hit || ok;
  }
  return hit;
}

__device__ __forceinline__ Key32 load_key(const uint8_t* tile, uint32_t j, int lane) {
  const uint4 a = lane_word(tile, 2 * j, lane);
  const uint4 b = lane_word(tile, 2 * j + 1, lane);
  Key32 k;
  k.q[0] = (uint64_t)a.x | ((uint64_t)a.y << 32);
  k.q[1] = (uint64_t)a.z | ((uint64_t)a.w << 32);
  k.q[2] = (uint64_t)b.x | ((uint64_t)b.y << 32);
  k.q[3] = (uint64_t)b.z | ((uint64_t)b.w << 32);
  k.q[4] = k.q[5] = k.q[6] = k.q[7] = 0;
  return k;
}

__device__ __forceinline__ void pattern_words(const GrepParams& p, uint64_t* pw, uint64_t* pm) {
#pragma unroll
  for (int b = 0; b < 4; ++b) {
    uint64_t w = 0, m = 0;
    for (int i = 0; i < 8; ++i) {
      const int x = 8 * b + i;
      if (x < (int)p.plen) { w |= (uint64_t)p.pat[x] << (8 * i); m |= 0xffull << (8 * i); }
    }
    pw[b] = w;
    pm[b] = m;
  }
}

__device__ __forceinline__ uint32_t block_sum(uint32_t v, uint32_t* sh) {
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  v = __reduce_add_sync(kFull, v);
  if (lane == 0) sh[wid] = v;
  __syncthreads();
  uint32_t s = 0;
  if (threadIdx.x == 0)
    for (int i = 0; i < (int)(blockDim.x >> 5); ++i) s += sh[i];
  return s;
}

__global__ void __launch_bounds__(256) k_grep_count(Chunk c, const uint8_t* __restrict__ stage,
                                                    const LaneDesc* __restrict__ lanes,
                                                    const uint64_t* __restrict__ tile_base, GrepParams p,
                                                    uint32_t* __restrict__ blkcnt) {
  __shared__ uint32_t sh[8];
  uint64_t pw[4], pm[4];
  pattern_words(p, pw, pm);
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
  uint32_t cnt = 0;
  if (t < c.L) {
    const LaneDesc d = lanes[t];
    const uint8_t* tile = stage + tile_base[t >> 5];
    for (uint32_t j = 0; j < d.nrec; ++j) cnt += grep_match(load_key(tile, j, t & 31), p, pw, pm);
  }
  const uint32_t s = block_sum(cnt, sh);
  if (threadIdx.x == 0) blkcnt[blockIdx.x] = s;
}

__global__ void __launch_bounds__(1024) k_grep_scan(uint32_t* __restrict__ blkcnt, uint32_t nblk,
                                                    unsigned long long* cursor, unsigned long long* blkbase,
                                                    unsigned long long* chunk_run) {
  __shared__ unsigned long long warp_sums[32];
  __shared__ unsigned long long carry;
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  // the chunk's match count, then its run in the pool: [base, base + total)
  unsigned long long part = 0;
  for (uint32_t i = threadIdx.x; i < nblk; i += 1024) part += blkcnt[i];
  part = __reduce_add_sync(kFull, (unsigned)part);
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
  for (uint32_t base = 0; base < nblk; base += 1024) {
    const uint32_t i = base + threadIdx.x;
    const unsigned long long v = i < nblk ? blkcnt[i] : 0;
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
    if (i < nblk) blkbase[i] = excl;
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

__global__ void __launch_bounds__(256) k_grep_write(Chunk c, const uint8_t* __restrict__ stage,
                                                    const LaneDesc* __restrict__ lanes,
                                                    const uint64_t* __restrict__ tile_base, GrepParams p,
                                                    const unsigned long long* __restrict__ blkbase,
                                                    uint64_t* __restrict__ out, int* err) {
  __shared__ uint32_t warp_tot[8];
  uint64_t pw[4], pm[4];
  pattern_words(p, pw, pm);
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  LaneDesc d{0, 0, 0};
  const uint8_t* tile = nullptr;
  uint32_t cnt = 0;
  if (t < c.L) {
    d = lanes[t];
    tile = stage + tile_base[t >> 5];
    for (uint32_t j = 0; j < d.nrec; ++j) cnt += grep_match(load_key(tile, j, lane), p, pw, pm);
  }
  if (__syncthreads_or(cnt) == 0) return;  // most blocks of a 1%-selective filter
  uint32_t x = cnt;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(kFull, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) warp_tot[wid] = x;
  __syncthreads();
  uint32_t before = 0;
  for (int i = 0; i < wid; ++i) before += warp_tot[i];
  unsigned long long pos = blkbase[blockIdx.x] + before + x - cnt;
  if (cnt) {
    for (uint32_t j = 0; j < d.nrec; ++j) {
      if (grep_match(load_key(tile, j, lane), p, pw, pm)) {
        if (pos < p.cap) out[pos] = p.first_index + d.first + j;
        else atomicOr(err, kErrOutOverflow);
        ++pos;
      }
    }
  }
}

// ------------------------------------------------------------------------------------------
// C5 group-by: records {u32 key, u32 qty, f64 amount} staged one word per record.
// Block-private shared-memory table (count, qty, amount), flushed once per block.

__global__ void __launch_bounds__(256) k_groupby(Chunk c, const uint8_t* __restrict__ stage,
                                                 const LaneDesc* __restrict__ lanes,
                                                 const uint64_t* __restrict__ tile_base, uint32_t G,
                                                 unsigned long long* gcount, unsigned long long* gqty,
                                                 double* gamount, int* err) {
  extern __shared__ unsigned char smem_raw[];
  double* s_amt = reinterpret_cast<double*>(smem_raw);
  unsigned int* s_cnt = reinterpret_cast<unsigned int*>(s_amt + G);
  unsigned int* s_qty = s_cnt + G;
  for (uint32_t g = threadIdx.x; g < G; g += blockDim.x) { s_amt[g] = 0.0; s_cnt[g] = 0; s_qty[g] = 0; }
  __syncthreads();
  for (uint32_t t = blockIdx.x * blockDim.x + threadIdx.x; t - threadIdx.x < c.L; t += gridDim.x * blockDim.x) {
    if (t < c.L) {
      const LaneDesc d = lanes[t];
      const uint8_t* tile = stage + tile_base[t >> 5];
      for (uint32_t j = 0; j < d.nrec; ++j) {
        const uint4 v = lane_word(tile, j, t & 31);
        const uint32_t key = v.x;
        if (key >= G) { atomicOr(err, kErrKeyRange); continue; }
        const double amt = __hiloint2double((int)v.w, (int)v.z);
        atomicAdd(&s_cnt[key], 1u);
        atomicAdd(&s_qty[key], v.y);
        atomicAdd(&s_amt[key], amt);
      }
    }
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

__global__ void __launch_bounds__(256) k_kmeans(Chunk c, const uint8_t* __restrict__ stage,
                                                const LaneDesc* __restrict__ lanes,
                                                const uint64_t* __restrict__ tile_base,
                                                const float* __restrict__ mu, uint32_t K, uint64_t first_index,
                                                unsigned long long* gcount, double* gsum,
                                                unsigned long long* gchk, int32_t* __restrict__ cid_out) {
  extern __shared__ unsigned char smem_raw[];
  double* s_sum = reinterpret_cast<double*>(smem_raw);          // K*16
  float* s_mu = reinterpret_cast<float*>(s_sum + (size_t)K * 16);  // K*16
  unsigned int* s_cnt = reinterpret_cast<unsigned int*>(s_mu + (size_t)K * 16);
  for (uint32_t i = threadIdx.x; i < K * 16; i += blockDim.x) { s_sum[i] = 0.0; s_mu[i] = mu[i]; }
  for (uint32_t i = threadIdx.x; i < K; i += blockDim.x) s_cnt[i] = 0;
  __syncthreads();
  unsigned long long chk = 0;
  for (uint32_t t = blockIdx.x * blockDim.x + threadIdx.x; t - threadIdx.x < c.L; t += gridDim.x * blockDim.x) {
    if (t >= c.L) continue;
    const LaneDesc d = lanes[t];
    const uint8_t* tile = stage + tile_base[t >> 5];
    for (uint32_t j = 0; j < d.nrec; ++j) {
      float x[16];
#pragma unroll
      for (int w = 0; w < 4; ++w) {
        const uint4 v = lane_word(tile, 4 * j + w, t & 31);
        x[4 * w + 0] = __uint_as_float(v.x);
        x[4 * w + 1] = __uint_as_float(v.y);
        x[4 * w + 2] = __uint_as_float(v.z);
        x[4 * w + 3] = __uint_as_float(v.w);
      }
      uint32_t best = 0;
      float bestd = 0.0f;
      for (uint32_t k = 0; k < K; ++k) {
        float acc = 0.0f;
#pragma unroll
        for (int q = 0; q < 16; ++q) {
          const float df = __fsub_rn(x[q], s_mu[k * 16 + q]);
          acc = __fmaf_rn(df, df, acc);
        }
        if (k == 0 || acc < bestd) { bestd = acc; best = k; }
      }
      atomicAdd(&s_cnt[best], 1u);
#pragma unroll
      for (int q = 0; q < 16; ++q) atomicAdd(&s_sum[best * 16 + q], (double)x[q]);
      chk += mix64(((first_index + d.first + j) << 8) ^ (uint64_t)best);
      if (cid_out) cid_out[d.first + j - c.lo] = (int32_t)best;
    }
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) chk += __shfl_xor_sync(kFull, chk, o);  // wraps mod 2^64
  __syncthreads();
  for (uint32_t i = threadIdx.x; i < K * 16; i += blockDim.x)
    if (s_sum[i] != 0.0) atomicAdd(&gsum[i], s_sum[i]);
  for (uint32_t i = threadIdx.x; i < K; i += blockDim.x)
    if (s_cnt[i]) atomicAdd(&gcount[i], (unsigned long long)s_cnt[i]);
  if ((threadIdx.x & 31) == 0) atomicAdd(gchk, chk);
}

}  // namespace

void launch_wc(const Chunk& c, const uint8_t* stage, const LaneDesc* lanes, const uint64_t* tile_base,
               const uint64_t* meta, uint64_t rec_size, WcEntry* table, uint64_t mask, unsigned long long* used,
               int* err, cudaStream_t s) {
  constexpr int kSub = 8;  // sub-threads per 256-B lane (sweep: 2/4/8/16, profiles/r01_wc_sweep.md)
  const uint32_t grid = (c.L * kSub + kWcBlock - 1) / kWcBlock;
  k_wc<kSub><<<grid, kWcBlock, 0, s>>>(c, stage, lanes, tile_base, meta, rec_size, table, mask, used, err);
}

void launch_wc_compact(const WcEntry* table, uint64_t slots, unsigned long long* n_out, uint64_t* off,
                       uint32_t* len, uint64_t* cnt, uint64_t cap, cudaStream_t s) {
  k_wc_compact<<<148 * 4, 256, 0, s>>>(table, slots, n_out, off, len, cnt, cap);
}

void launch_grep(const Chunk& c, const uint8_t* stage, const LaneDesc* lanes, const uint64_t* tile_base,
                 const GrepParams& p, uint32_t* blkcnt, unsigned long long* cursor, unsigned long long* blkbase,
                 unsigned long long* chunk_run, uint64_t* out_idx, int* err, cudaStream_t s) {
  const uint32_t nblk = (c.L + 255) / 256;
  k_grep_count<<<nblk, 256, 0, s>>>(c, stage, lanes, tile_base, p, blkcnt);
  k_grep_scan<<<1, 1024, 0, s>>>(blkcnt, nblk, cursor, blkbase, chunk_run);
  k_grep_write<<<nblk, 256, 0, s>>>(c, stage, lanes, tile_base, p, blkbase, out_idx, err);
}

void launch_grep_order(const unsigned long long* runs, uint32_t C, const uint64_t* pool, uint64_t* out, uint64_t cap,
                       cudaStream_t s) {
  if (C) k_grep_order<<<C, 256, 0, s>>>(runs, C, pool, out, cap);
}

size_t groupby_smem(uint32_t G) { return (size_t)G * 16; }

void launch_groupby(const Chunk& c, const uint8_t* stage, const LaneDesc* lanes, const uint64_t* tile_base,
                    uint32_t G, unsigned long long* count, unsigned long long* qty, double* amount, int* err,
                    int grid, cudaStream_t s) {
  k_groupby<<<grid, 256, groupby_smem(G), s>>>(c, stage, lanes, tile_base, G, count, qty, amount, err);
}

size_t kmeans_smem(uint32_t K) { return (size_t)K * 16 * 8 + (size_t)K * 16 * 4 + (size_t)K * 4; }

void launch_kmeans(const Chunk& c, const uint8_t* stage, const LaneDesc* lanes, const uint64_t* tile_base,
                   const float* mu, uint32_t K, uint64_t first_index, unsigned long long* count, double* sum,
                   unsigned long long* chk, int32_t* cid_out, int grid, cudaStream_t s) {
  k_kmeans<<<grid, 256, kmeans_smem(K), s>>>(c, stage, lanes, tile_base, mu, K, first_index, count, sum, chk,
                                              cid_out);
}

cudaError_t configure_compute_kernels() {
  cudaError_t e = cudaFuncSetAttribute(k_groupby, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  if (e != cudaSuccess) return e;
  return cudaFuncSetAttribute(k_kmeans, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
}

}  // namespace bk
