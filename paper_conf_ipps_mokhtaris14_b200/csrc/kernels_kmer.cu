// kernels_kmer.cu — f4, the second workload family: k-mer counting over fixed-length DNA read
// records (the paper's DNA assembly builds a k-mer hash table; Table I P:927:
// fixed-length records, 36% read). Stage 1-3 stage only the sequence field (FIELD access); here
// each thread walks its lane's reads base by base (the warp in lockstep: reads have one length),
// rolls the 2-bit k-mer (A=0 C=1 G=2 T=3; any other byte breaks the window) and counts it in an
// exact-key open-addressing table (key = k-mer + 1, no hashing collisions in identity), in two
// phases (below).
#include "bk_internal.cuh"

#include <algorithm>

namespace bk {
namespace {

constexpr unsigned kFull = 0xffffffffu;

// inverse of mix64: each xorshift undone by its own series, each odd multiplier by its inverse mod 2^64
__device__ __forceinline__ uint64_t unmix64(uint64_t x) {
  x ^= (x >> 31) ^ (x >> 62);
  x *= 0x319642b2d24d8ec3ULL;
  x ^= (x >> 27) ^ (x >> 54);
  x *= 0x96de1b173f119089ULL;
  x ^= (x >> 30) ^ (x >> 60);
  return x;
}

// ---- two-phase counting (round 2): the table is split into R = 2^rb regions of S slots; a k-mer's
// region is the top rb bits of h = mix64(key), its home slot the low bits. mix64 (the splitmix64
// finalizer) is a bijection with mix64(0) = 0, so buckets and table slots hold h itself: equal h is
// equal key, h != 0 marks an occupied slot, the hash is computed once per window (phase A), and the
// k-mer is recovered by unmix64 only when a distinct entry is emitted. Phase A (stage 4, per chunk)
// appends every k-mer window's key to its region's bucket in HBM (one L2 atomic on the bucket cursor
// + one 8-B store; the L2 merges a bucket's consecutive appends into whole sectors). Phase B (flush)
// gives each region to one CTA: the region is loaded into shared memory (S x 12 B <= 96 KiB), the
// bucket's keys are counted with shared-memory atomics and the region is written back — DRAM traffic
// ~24 B per k-mer (8 B appended, 8 B read back, the table read and written once per flush) instead of
// a random 16-B table entry per k-mer (~146 B of DRAM per update measured in round 1). A bucket that
// fills up sends the rest of its keys straight to the region in HBM (same slots), so any input is
// counted exactly.

__device__ __forceinline__ void region_insert(KmerEntry* region, uint64_t smask, unsigned long long key,
                                              unsigned long long cnt, int* err) {
  // key = mix64(k-mer + 1) (nonzero); callers mark the region dirty: its HBM copy now holds counts a
  // flush must load
  uint64_t slot = key & smask;
  for (uint64_t probe = 0; probe <= smask; ++probe, slot = (slot + 1) & smask) {
    unsigned long long k = *reinterpret_cast<volatile unsigned long long*>(&region[slot].key);
    if (k == 0) k = atomicCAS(&region[slot].key, 0ull, key);
    if (k == 0 || k == key) {
      atomicAdd(&region[slot].count, cnt);
      return;
    }
  }
  atomicOr(err, kErrTableFull);
}

// Block-level bucketing (phase A and the coarse -> fine split): a block stages up to kStep keys in
// shared memory, sorts them by bin (shared-memory histogram + scan), reserves each bin's run in its
// global bucket with ONE atomic per (block step, bin) and writes the runs coalesced. Keys of a full
// bucket go to their table region in HBM directly (exact for any input).
constexpr int kBinThreads = 256;
constexpr uint32_t kStep = kBinThreads * 16;   // keys per block step (16 per thread: one staged word)
constexpr uint32_t kMaxBins = 256;

struct BinSmem {
  unsigned int hist[kMaxBins], boff[kMaxBins + 1], gpos[kMaxBins];
  unsigned long long key[kStep];
  unsigned short bin[kStep];
};

// One block step: thread-local keys (okm bits of key[16], their bins in bn[16]) -> buckets
// gbuf[bin * gcap ...] (cursors gcur[bin]); `region_of(key)` / `rbase` locate a key's table region
// for the fallback. Every thread of the block must call it.
template <class RegionOf>
__device__ __forceinline__ void bin_step(BinSmem& sm, uint32_t nbins, const unsigned long long* key, const uint32_t* bn,
                                         uint32_t okm, unsigned long long* gbuf, unsigned int* gcur, uint32_t gcap,
                                         KmerEntry* table, uint64_t smask, unsigned char* dirty, int* err,
                                         RegionOf&& region_of) {
  const uint32_t tid = threadIdx.x;
  for (uint32_t i = tid; i < nbins; i += blockDim.x) sm.hist[i] = 0;
  __syncthreads();
  unsigned lp[16];
#pragma unroll
  for (int b = 0; b < 16; ++b) lp[b] = (okm >> b & 1) ? atomicAdd(&sm.hist[bn[b]], 1u) : 0u;
  __syncthreads();
  if (tid < 32) {   // exclusive scan of the histogram (nbins <= 256: 8 per lane)
    unsigned v[8], sum = 0;
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      const uint32_t i = tid * 8 + q;
      v[q] = i < nbins ? sm.hist[i] : 0u;
      sum += v[q];
    }
    unsigned incl = sum;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const unsigned y = __shfl_up_sync(kFull, incl, o);
      if (tid >= (uint32_t)o) incl += y;
    }
    unsigned run = incl - sum;
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      const uint32_t i = tid * 8 + q;
      if (i < nbins) sm.boff[i] = run;
      run += v[q];
    }
    if (tid == 31) sm.boff[nbins] = incl;
  }
  for (uint32_t i = tid; i < nbins; i += blockDim.x) sm.gpos[i] = sm.hist[i] ? atomicAdd(&gcur[i], sm.hist[i]) : 0u;
  __syncthreads();
#pragma unroll
  for (int b = 0; b < 16; ++b) {
    if (!(okm >> b & 1)) continue;
    const uint32_t i = sm.boff[bn[b]] + lp[b];
    sm.key[i] = key[b];
    sm.bin[i] = (unsigned short)bn[b];
  }
  __syncthreads();
  const uint32_t total = sm.boff[nbins];
  for (uint32_t i = tid; i < total; i += blockDim.x) {
    const uint32_t bi = sm.bin[i];
    const unsigned long long kk = sm.key[i];
    const uint64_t pos = (uint64_t)sm.gpos[bi] + (i - sm.boff[bi]);
    if (pos < gcap) {
      gbuf[(size_t)bi * gcap + pos] = kk;
    } else {   // bucket full: straight into the key's region in HBM
      const uint32_t r = region_of(kk);
      region_insert(table + (size_t)r * (smask + 1), smask, kk, 1ull, err);
      dirty[r] = 1;
    }
  }
  __syncthreads();
}

// Phase A (stage 4, per chunk): every k-mer window of the lane's reads -> h = mix64(k-mer + 1) -> its
// coarse bin (the top cb bits of h; cb == rb: the bins are the regions' buckets themselves)
__global__ void __launch_bounds__(kBinThreads) k_kmer_bin(Chunk c, const uint8_t* __restrict__ stage,
                                                          const LaneDesc* __restrict__ lanes,
                                                          const uint64_t* __restrict__ tile_base, uint32_t k,
                                                          uint32_t seq_words, KmerEntry* table, uint32_t rb,
                                                          uint32_t cb, uint64_t smask,
                                                          unsigned long long* __restrict__ gbuf,
                                                          unsigned int* __restrict__ gcur, uint32_t gcap,
                                                          unsigned char* __restrict__ dirty,
                                                          unsigned long long* total, int* err) {
  __shared__ BinSmem sm;
  __shared__ uint32_t s_rmax;
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
  const int lane = threadIdx.x & 31;
  const bool live = t < c.L;
  LaneDesc d{0, 0, 0};
  if (live) d = lanes[t];
  const uint8_t* tile = stage + (live ? tile_base[t >> 5] : 0);
  if (threadIdx.x == 0) s_rmax = 0;
  __syncthreads();
  atomicMax(&s_rmax, d.nrec);
  __syncthreads();
  const uint32_t R = s_rmax;   // block-uniform trip count (the steps synchronise the block)
  const uint64_t kmask = k == 32 ? ~0ull : ((1ull << (2 * k)) - 1);
  auto region_of = [&](unsigned long long h) -> uint32_t { return rb ? (uint32_t)(h >> (64 - rb)) : 0u; };
  unsigned long long mine = 0;
  for (uint32_t j = 0; j < R; ++j) {
    const bool rec = j < d.nrec;
    uint64_t v = 0;
    uint32_t valid = 0;
    for (uint32_t w = 0; w < seq_words; ++w) {
      uint4 q = make_uint4(0, 0, 0, 0);
      if (rec) q = *reinterpret_cast<const uint4*>(tile + ((size_t)(j * seq_words + w) * 32 + lane) * 16);
      const uint32_t wd[4] = {q.x, q.y, q.z, q.w};
      unsigned long long key[16];
      uint32_t bn[16];
      uint32_t okm = 0;
#pragma unroll
      for (int b = 0; b < 16; ++b) {
        const uint32_t ch = (wd[b >> 2] >> (8 * (b & 3))) & 0xff;
        const int code = ch == 'A' ? 0 : ch == 'C' ? 1 : ch == 'G' ? 2 : ch == 'T' ? 3 : -1;
        if (code < 0) {
          valid = 0;
          v = 0;
        } else {
          v = ((v << 2) | (uint64_t)code) & kmask;
          ++valid;
        }
        key[b] = mix64(v + 1);
        bn[b] = cb ? (uint32_t)(key[b] >> (64 - cb)) : 0u;
        if (rec && valid >= k) okm |= 1u << b;
      }
      mine += __popc(okm);
      bin_step(sm, 1u << cb, key, bn, okm, gbuf, gcur, gcap, table, smask, dirty, err, region_of);
    }
  }
  for (int o = 16; o; o >>= 1) mine += __shfl_down_sync(kFull, mine, o);
  if (lane == 0 && mine) atomicAdd(total, mine);
}

// Flush, first half (cb < rb): coarse bin b's keys -> the buckets of its 2^(rb-cb) regions. Grid
// (slices, coarse bins); resets the coarse cursor when its last slice is done (a per-bin counter).
__global__ void __launch_bounds__(kBinThreads) k_kmer_split(const unsigned long long* __restrict__ cbuf,
                                                            unsigned int* __restrict__ ccur, uint32_t ccap,
                                                            unsigned int* __restrict__ cdone, uint32_t rb, uint32_t cb,
                                                            unsigned long long* __restrict__ fbuf,
                                                            unsigned int* __restrict__ fcur, uint32_t fcap,
                                                            KmerEntry* table, uint64_t smask,
                                                            unsigned char* __restrict__ dirty, int* err) {
  __shared__ BinSmem sm;
  const uint32_t b = blockIdx.y, nslice = gridDim.x, sl = blockIdx.x;
  const uint32_t n = min(ccur[b], ccap);
  const uint32_t lo = (uint32_t)((uint64_t)n * sl / nslice), hi = (uint32_t)((uint64_t)n * (sl + 1) / nslice);
  const uint32_t fb = rb - cb;   // fine bits within the coarse bin
  const unsigned long long* keys = cbuf + (size_t)b * ccap;
  auto region_of = [&](unsigned long long h) -> uint32_t { return (uint32_t)(h >> (64 - rb)); };
  for (uint32_t base = lo; base < hi; base += kStep) {
    unsigned long long key[16];
    uint32_t bn[16];
    uint32_t okm = 0;
#pragma unroll
    for (int q = 0; q < 16; ++q) {
      const uint32_t i = base + q * blockDim.x + threadIdx.x;
      key[q] = i < hi ? keys[i] : 0ull;
      bn[q] = i < hi ? (uint32_t)(key[q] >> (64 - rb)) & ((1u << fb) - 1) : 0u;
      if (i < hi) okm |= 1u << q;
    }
    bin_step(sm, 1u << fb, key, bn, okm, fbuf + (size_t)b * (1ull << fb) * fcap, fcur + ((size_t)b << fb), fcap,
             table, smask, dirty, err, region_of);
  }
  __syncthreads();
  if (threadIdx.x == 0 && atomicAdd(&cdone[b], 1u) + 1 == nslice) {   // the bin's last slice: reset it
    ccur[b] = 0;
    cdone[b] = 0;
  }
}

// one CTA per region: the region's keys -> shared memory (loaded only if its HBM copy holds counts: a
// direct insert or an earlier flush; else zeros), count its bucket with shared-memory atomics, reset
// the cursor; then either write the region back (a mid-run flush) or, on the final flush, emit its
// occupied entries straight to the result arrays (no write-back, no separate compaction pass). Shared
// memory holds 8-B keys and 32-bit counts of THIS flush (12 B per slot: a 64-bit shared atomicAdd
// compiles to a CAS loop, a 32-bit one is native, and 2 CTAs fit per SM); the region's earlier
// 64-bit count is added back from HBM when it is written back or emitted, so counts stay exact.
__global__ void __launch_bounds__(512, 2) k_kmer_flush(KmerEntry* table, uint32_t rb, uint64_t smask,
                                                      const unsigned long long* __restrict__ bbuf,
                                                      unsigned int* __restrict__ bcur, uint32_t bcap,
                                                      unsigned char* __restrict__ dirty, int final_flush,
                                                      uint64_t* __restrict__ out_kmer, uint64_t* __restrict__ out_cnt,
                                                      uint64_t ocap, unsigned long long* n_out, int* err) {
  extern __shared__ __align__(16) unsigned char km_smem[];
  __shared__ unsigned int s_wsum[16];
  __shared__ unsigned long long s_base;
  const uint32_t r = blockIdx.x;
  const uint64_t S = smask + 1;
  unsigned long long* skey = reinterpret_cast<unsigned long long*>(km_smem);
  unsigned int* scnt = reinterpret_cast<unsigned int*>(skey + S);
  KmerEntry* region = table + (size_t)r * S;
  const uint32_t n = min(bcur[r], bcap);
  const bool had = dirty[r] != 0;
  if (n == 0 && !final_flush) {   // nothing appended: the region in HBM is already current
    __syncthreads();
    if (threadIdx.x == 0) bcur[r] = 0;
    return;
  }
  if (n == 0 && !had) return;   // final flush of an empty region: nothing to emit
  for (uint64_t i = threadIdx.x; i < S; i += blockDim.x) {
    skey[i] = had ? region[i].key : 0ull;
    scnt[i] = 0u;
  }
  __syncthreads();
  const unsigned long long* keys = bbuf + (size_t)r * bcap;
  auto count = [&](unsigned long long key) {
    uint64_t slot = key & smask;
    for (uint64_t probe = 0; probe <= smask; ++probe, slot = (slot + 1) & smask) {
      unsigned long long kk = skey[slot];
      if (kk == 0) kk = atomicCAS(&skey[slot], 0ull, key);
      if (kk == 0 || kk == key) {
        atomicAdd(&scnt[slot], 1u);
        return;
      }
    }
    atomicOr(err, kErrTableFull);
  };
  constexpr uint32_t kIlp = 4;   // bucket keys in flight per thread (the loop is load-latency bound)
  uint32_t ki = threadIdx.x;
  for (; ki + (kIlp - 1) * blockDim.x < n; ki += kIlp * blockDim.x) {
    unsigned long long kq[kIlp];
#pragma unroll
    for (uint32_t q = 0; q < kIlp; ++q) kq[q] = __ldcs(keys + ki + q * blockDim.x);
#pragma unroll
    for (uint32_t q = 0; q < kIlp; ++q) count(kq[q]);
  }
  for (; ki < n; ki += blockDim.x) count(__ldcs(keys + ki));
  __syncthreads();
  if (!final_flush) {
    for (uint64_t i = threadIdx.x; i < S; i += blockDim.x) {
      const unsigned long long kk = skey[i];
      if (kk == 0) continue;   // empty here is empty in HBM too (the region was loaded or zero)
      region[i].key = kk;
      region[i].count = (had ? region[i].count : 0ull) + scnt[i];
    }
    if (threadIdx.x == 0) {
      bcur[r] = 0;
      dirty[r] = 1;
    }
    return;
  }
  // emit, coalesced: the region's occupied slots in slot order go to consecutive result positions
  // (one atomic per region for the base; per 512-slot stripe a block-wide ballot scan), so a warp's
  // stores are contiguous — the result arrays may be mapped host memory written over PCIe
  const uint32_t lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = blockDim.x / 32;
  uint32_t mine = 0;
  for (uint64_t i = threadIdx.x; i < S; i += blockDim.x) mine += skey[i] != 0;
  for (int o = 16; o; o >>= 1) mine += __shfl_xor_sync(kFull, mine, o);
  if (lane == 0) s_wsum[wid] = mine;
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned int acc = 0;
    for (uint32_t w = 0; w < nw; ++w) acc += s_wsum[w];
    s_base = acc ? atomicAdd(n_out, (unsigned long long)acc) : 0ull;
  }
  __syncthreads();
  unsigned long long base = s_base;
  for (uint64_t i0 = 0; i0 < S; i0 += blockDim.x) {
    const uint64_t i = i0 + threadIdx.x;
    const unsigned long long kk = i < S ? skey[i] : 0ull;
    const unsigned occ = __ballot_sync(kFull, kk != 0);
    __syncthreads();   // the previous stripe's s_wsum reads are done
    if (lane == 0) s_wsum[wid] = __popc(occ);
    __syncthreads();
    unsigned before = 0, total = 0;
    for (uint32_t w = 0; w < nw; ++w) {
      const unsigned v = s_wsum[w];
      before += w < wid ? v : 0u;
      total += v;
    }
    if (kk != 0) {
      const unsigned long long p = base + before + __popc(occ & ((1u << lane) - 1));
      if (p < ocap) {
        out_kmer[p] = unmix64(kk) - 1;
        out_cnt[p] = (had ? region[i].count : 0ull) + scnt[i];
      }
    }
    base += total;
  }
  if (threadIdx.x == 0) bcur[r] = 0;
}

}  // namespace

size_t kmer_flush_smem(uint64_t region_slots) { return (size_t)region_slots * 12; }   // 8-B key + 32-bit count

void launch_kmer_bin(const Chunk& c, const uint8_t* stage, const LaneDesc* lanes, const uint64_t* tile_base,
                     uint32_t k, uint32_t seq_words, KmerEntry* table, uint32_t rb, uint32_t cb, uint64_t region_slots,
                     unsigned long long* gbuf, unsigned int* gcur, uint32_t gcap, unsigned char* dirty,
                     unsigned long long* total, int* err, cudaStream_t s) {
  k_kmer_bin<<<(c.L + kBinThreads - 1) / kBinThreads, kBinThreads, 0, s>>>(c, stage, lanes, tile_base, k, seq_words,
                                                                        table, rb, cb, region_slots - 1, gbuf, gcur,
                                                                        gcap, dirty, total, err);
}

void launch_kmer_split(const unsigned long long* cbuf, unsigned int* ccur, uint32_t ccap, unsigned int* cdone,
                       uint32_t rb, uint32_t cb, unsigned long long* fbuf, unsigned int* fcur, uint32_t fcap,
                       KmerEntry* table, uint64_t region_slots, unsigned char* dirty, int* err, cudaStream_t s) {
  const uint32_t slices = std::max(1, 2 * device_sms() / (1 << cb) + 1);
  k_kmer_split<<<dim3(slices, 1u << cb), kBinThreads, 0, s>>>(cbuf, ccur, ccap, cdone, rb, cb, fbuf, fcur, fcap, table,
                                                             region_slots - 1, dirty, err);
}

void launch_kmer_flush(KmerEntry* table, uint32_t rb, uint64_t region_slots, const unsigned long long* bbuf,
                       unsigned int* bcur, uint32_t bcap, unsigned char* dirty, int final_flush, uint64_t* out_kmer,
                       uint64_t* out_cnt, uint64_t ocap, unsigned long long* n_out, int* err, cudaStream_t s) {
  k_kmer_flush<<<1u << rb, 512, kmer_flush_smem(region_slots), s>>>(table, rb, region_slots - 1, bbuf, bcur, bcap,
                                                                      dirty, final_flush, out_kmer, out_cnt, ocap,
                                                                      n_out, err);
}

cudaError_t configure_kmer_kernels() {
  return cudaFuncSetAttribute((const void*)k_kmer_flush, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
}

}  // namespace bk
