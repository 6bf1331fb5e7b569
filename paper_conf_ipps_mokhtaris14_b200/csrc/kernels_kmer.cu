// kernels_kmer.cu — f4, the second workload family: k-mer counting over fixed-length DNA read
// records (the paper's DNA assembly builds a k-mer hash table; Table I P:927:
// fixed-length records, 36% read). Stage 1-3 stage only the sequence field (FIELD access); here
// each thread walks its lane's reads base by base (the warp in lockstep: reads have one length),
// rolls the 2-bit k-mer (A=0 C=1 G=2 T=3; any other byte breaks the window) and counts it in an
// exact-key open-addressing table (key = k-mer + 1, no hashing collisions in identity), in two
// phases (below).
#include "bk_internal.cuh"

namespace bk {
namespace {

constexpr unsigned kFull = 0xffffffffu;

// ---- two-phase counting (round 2): the table is split into R = 2^rb regions of S slots; a k-mer's
// region is the top rb bits of mix64(key), its home slot the low bits. Phase A (stage 4, per chunk)
// appends every k-mer window's key to its region's bucket in HBM (one L2 atomic on the bucket cursor
// + one 8-B store; the L2 merges a bucket's consecutive appends into whole sectors). Phase B (flush)
// gives each region to one CTA: the region is loaded into shared memory (S x 16 B <= 128 KiB), the
// bucket's keys are counted with shared-memory atomics and the region is written back — DRAM traffic
// ~24 B per k-mer (8 B appended, 8 B read back, the table read and written once per flush) instead of
// a random 16-B table entry per k-mer (~146 B of DRAM per update measured in round 1). A bucket that
// fills up sends the rest of its keys straight to the region in HBM (same slots), so any input is
// counted exactly.

__device__ __forceinline__ void region_insert(KmerEntry* region, uint64_t smask, uint64_t h,
                                              unsigned long long key, unsigned long long cnt, int* err) {
  // (callers mark the region dirty: its HBM copy now holds counts a flush must load)
  uint64_t slot = h & smask;
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

__global__ void __launch_bounds__(256) k_kmer_scatter(Chunk c, const uint8_t* __restrict__ stage,
                                                      const LaneDesc* __restrict__ lanes,
                                                      const uint64_t* __restrict__ tile_base, uint32_t k,
                                                      uint32_t seq_words, KmerEntry* table, uint32_t rb,
                                                      uint64_t smask, unsigned long long* __restrict__ bbuf,
                                                      unsigned int* __restrict__ bcur, uint32_t bcap,
                                                      unsigned char* __restrict__ dirty,
                                                      unsigned long long* total, int* err) {
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= c.L) return;  // whole warps
  const int lane = t & 31;
  const LaneDesc d = lanes[t];
  const uint8_t* tile = stage + tile_base[t >> 5];
  const uint32_t R = __reduce_max_sync(kFull, d.nrec);
  const uint64_t kmask = k == 32 ? ~0ull : ((1ull << (2 * k)) - 1);
  unsigned long long mine = 0;
  for (uint32_t j = 0; j < R; ++j) {
    const bool rec = j < d.nrec;
    uint64_t v = 0;
    uint32_t valid = 0;
    for (uint32_t w = 0; w < seq_words; ++w) {
      uint4 q = make_uint4(0, 0, 0, 0);
      if (rec) q = *reinterpret_cast<const uint4*>(tile + ((size_t)(j * seq_words + w) * 32 + lane) * 16);
      const uint32_t wd[4] = {q.x, q.y, q.z, q.w};
      // the word's up to 16 k-mers first, then their 16 independent cursor atomics, then the stores:
      // one L2 round trip per 16 windows instead of one per window
      unsigned long long key[16];
      uint32_t bk[16];
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
        key[b] = v + 1;
        bk[b] = rb ? (uint32_t)(mix64(key[b]) >> (64 - rb)) : 0u;
        if (rec && valid >= k) okm |= 1u << b;
      }
      unsigned pos[16];
#pragma unroll
      for (int b = 0; b < 16; ++b) pos[b] = (okm >> b & 1) ? atomicAdd(&bcur[bk[b]], 1u) : 0u;
#pragma unroll
      for (int b = 0; b < 16; ++b) {
        if (!(okm >> b & 1)) continue;
        if (pos[b] < bcap) {
          bbuf[(size_t)bk[b] * bcap + pos[b]] = key[b];
        } else {   // bucket full: straight into the region in HBM
          region_insert(table + (size_t)bk[b] * (smask + 1), smask, mix64(key[b]), key[b], 1ull, err);
          dirty[bk[b]] = 1;
        }
      }
      mine += __popc(okm);
    }
  }
  mine = __reduce_add_sync(kFull, (unsigned)mine);
  if (lane == 0 && mine) atomicAdd(total, mine);
}

// one CTA per region: the region -> shared memory (loaded only if its HBM copy holds counts: a direct
// insert or an earlier flush; else zeros), count its bucket with shared-memory atomics, reset the
// cursor; then either write the region back (a mid-run flush) or, on the final flush, emit its
// occupied entries straight to the result arrays (no write-back, no separate compaction pass)
__global__ void __launch_bounds__(512) k_kmer_flush(KmerEntry* table, uint32_t rb, uint64_t smask,
                                                   const unsigned long long* __restrict__ bbuf,
                                                   unsigned int* __restrict__ bcur, uint32_t bcap,
                                                   unsigned char* __restrict__ dirty, int final_flush,
                                                   uint64_t* __restrict__ out_kmer, uint64_t* __restrict__ out_cnt,
                                                   uint64_t ocap, unsigned long long* n_out, int* err) {
  extern __shared__ __align__(16) unsigned char km_smem[];
  __shared__ unsigned int s_wsum[16];
  __shared__ unsigned long long s_base;
  KmerEntry* sreg = reinterpret_cast<KmerEntry*>(km_smem);
  const uint32_t r = blockIdx.x;
  const uint64_t S = smask + 1;
  KmerEntry* region = table + (size_t)r * S;
  const uint32_t n = min(bcur[r], bcap);
  const bool had = dirty[r] != 0;
  if (n == 0 && !final_flush) {   // nothing appended: the region in HBM is already current
    __syncthreads();
    if (threadIdx.x == 0) bcur[r] = 0;
    return;
  }
  if (n == 0 && !had) return;   // final flush of an empty region: nothing to emit
  for (uint64_t i = threadIdx.x; i < S; i += blockDim.x)
    reinterpret_cast<ulonglong2*>(sreg)[i] = had ? reinterpret_cast<const ulonglong2*>(region)[i] : make_ulonglong2(0, 0);
  __syncthreads();
  const unsigned long long* keys = bbuf + (size_t)r * bcap;
  for (uint32_t i = threadIdx.x; i < n; i += blockDim.x) {
    const unsigned long long key = keys[i];
    const uint64_t h = mix64(key);
    uint64_t slot = h & smask;
    bool done = false;
    for (uint64_t probe = 0; probe <= smask; ++probe, slot = (slot + 1) & smask) {
      unsigned long long kk = sreg[slot].key;
      if (kk == 0) kk = atomicCAS(&sreg[slot].key, 0ull, key);
      if (kk == 0 || kk == key) {
        atomicAdd(&sreg[slot].count, 1ull);
        done = true;
        break;
      }
    }
    if (!done) atomicOr(err, kErrTableFull);
  }
  __syncthreads();
  if (!final_flush) {
    for (uint64_t i = threadIdx.x; i < S; i += blockDim.x)
      reinterpret_cast<ulonglong2*>(region)[i] = reinterpret_cast<const ulonglong2*>(sreg)[i];
    if (threadIdx.x == 0) {
      bcur[r] = 0;
      dirty[r] = 1;
    }
    return;
  }
  // emit: every thread its slots i = tid + j*512 in order; block prefix of the occupied counts
  const uint32_t lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  uint32_t mine = 0;
  for (uint64_t i = threadIdx.x; i < S; i += blockDim.x) mine += sreg[i].key != 0;
  uint32_t incl = mine;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(kFull, incl, o);
    if (lane >= (uint32_t)o) incl += y;
  }
  if (lane == 31) s_wsum[wid] = incl;
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned int acc = 0;
    for (uint32_t w = 0; w < blockDim.x / 32; ++w) {
      const unsigned int v = s_wsum[w];
      s_wsum[w] = acc;
      acc += v;
    }
    s_base = acc ? atomicAdd(n_out, (unsigned long long)acc) : 0ull;
  }
  __syncthreads();
  unsigned long long p = s_base + s_wsum[wid] + incl - mine;
  for (uint64_t i = threadIdx.x; i < S; i += blockDim.x) {
    const KmerEntry e = sreg[i];
    if (e.key == 0) continue;
    if (p < ocap) {
      out_kmer[p] = e.key - 1;
      out_cnt[p] = e.count;
    }
    ++p;
  }
  if (threadIdx.x == 0) bcur[r] = 0;
}

}  // namespace

size_t kmer_flush_smem(uint64_t region_slots) { return (size_t)region_slots * sizeof(KmerEntry); }

void launch_kmer_scatter(const Chunk& c, const uint8_t* stage, const LaneDesc* lanes, const uint64_t* tile_base,
                         uint32_t k, uint32_t seq_words, KmerEntry* table, uint32_t rb, uint64_t region_slots,
                         unsigned long long* bbuf, unsigned int* bcur, uint32_t bcap, unsigned char* dirty,
                         unsigned long long* total, int* err, cudaStream_t s) {
  k_kmer_scatter<<<(c.L + 255) / 256, 256, 0, s>>>(c, stage, lanes, tile_base, k, seq_words, table, rb,
                                                    region_slots - 1, bbuf, bcur, bcap, dirty, total, err);
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
