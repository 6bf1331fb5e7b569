// kernels_partition.cu — C4 stable hash partition of {u64 key, u64 value} records into B buckets
// (the paper's "partition" class; bucket = mix64(key) >> (64-log2 B),
// DESIGN.md A14). Per chunk the output is the chunk's records in (bucket, record) order, so the
// global stable partition is the chunk-major concatenation of each bucket's runs.
//
// Records arrive in the warp-tile layout (16-B record = one word; lane t holds records
// [first_t, first_t + nrec_t)). Record order inside a tile is lane-major, so a warp walks its
// tile in record order 32 records at a time and ranks equal buckets with __match_any_sync.
//   K1 k_part_hist : block histogram of its contiguous tile range   -> hist[b][blk]
//   K2 k_part_cols : per bucket, exclusive scan over blocks          -> colpre[b][blk], total[b]
//   K3 k_part_base : exclusive scan of total over buckets            -> base[b], counts out
//   K4 k_part_scatter: base[b] + colpre[b][blk] + earlier tiles of the block + rank in tile
#include "bk_internal.cuh"

namespace bk {
namespace {

constexpr unsigned kFull = 0xffffffffu;
constexpr int kPB = 256;   // threads per block (8 warps; warp w takes tiles w, w+8, ... of the block range)

__device__ __forceinline__ uint32_t bucket_of(uint64_t key, int bits) {
  return bits ? (uint32_t)(mix64(key) >> (64 - bits)) : 0u;
}

struct TileWalk {  // maps tile-record index p -> (lane, word) via the warp's nrec prefix
  uint32_t incl, nrec;
  uint32_t total;
  __device__ void init(const LaneDesc& d, int lane) {
    nrec = d.nrec;
    incl = nrec;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(kFull, incl, o);
      if (lane >= o) incl += y;
    }
    total = __shfl_sync(kFull, incl, 31);
  }
  __device__ void locate(uint32_t p, int& t, uint32_t& j) const {
    t = 0;
#pragma unroll
    for (int step = 16; step; step >>= 1) {
      const uint32_t v = __shfl_sync(kFull, incl, t + step - 1);
      if (v <= p) t += step;
    }
    t = t > 31 ? 31 : t;
    const uint32_t it = __shfl_sync(kFull, incl, t), nt = __shfl_sync(kFull, nrec, t);
    j = p - (it - nt);
  }
};

__device__ __forceinline__ void block_tiles(uint32_t ntiles, uint32_t nblk, uint32_t blk, uint32_t& t0, uint32_t& t1) {
  const uint32_t per = (ntiles + nblk - 1) / nblk;
  t0 = min(ntiles, blk * per);
  t1 = min(ntiles, t0 + per);
}

__global__ void __launch_bounds__(kPB) k_part_hist(Chunk c, const uint8_t* __restrict__ stage,
                                                   const LaneDesc* __restrict__ lanes,
                                                   const uint64_t* __restrict__ tile_base, int bits,
                                                   uint32_t* __restrict__ hist) {
  extern __shared__ uint32_t sh[];
  const uint32_t B = 1u << bits;
  for (uint32_t b = threadIdx.x; b < B; b += blockDim.x) sh[b] = 0;
  __syncthreads();
  uint32_t t0, t1;
  block_tiles(c.ntiles, gridDim.x, blockIdx.x, t0, t1);
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (uint32_t ti = t0 + w; ti < t1; ti += kPB / 32) {
    const LaneDesc d = lanes[(size_t)ti * 32 + lane];
    const uint8_t* tile = stage + tile_base[ti];
    // every word of every lane is one record: count lane-locally, no ordering needed here
    for (uint32_t j = 0; j < d.nrec; ++j) {
      const uint4 v = *reinterpret_cast<const uint4*>(tile + ((size_t)j * 32 + lane) * 16);
      atomicAdd(&sh[bucket_of((uint64_t)v.x | ((uint64_t)v.y << 32), bits)], 1u);
    }
  }
  __syncthreads();
  for (uint32_t b = threadIdx.x; b < B; b += blockDim.x) hist[(size_t)b * gridDim.x + blockIdx.x] = sh[b];
}

// one block per bucket: colpre[b][blk] = sum_{blk' < blk} hist[b][blk'], total[b]
__global__ void __launch_bounds__(256) k_part_cols(const uint32_t* __restrict__ hist, uint32_t nblk,
                                                   uint32_t* __restrict__ colpre, unsigned long long* __restrict__ total) {
  __shared__ uint32_t ws[8];
  __shared__ uint32_t carry;
  const uint32_t b = blockIdx.x;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  for (uint32_t base = 0; base < nblk; base += 256) {
    const uint32_t i = base + threadIdx.x;
    const uint32_t v = i < nblk ? hist[(size_t)b * nblk + i] : 0;
    uint32_t x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(kFull, x, o);
      if (lane >= o) x += y;
    }
    if (lane == 31) ws[w] = x;
    __syncthreads();
    uint32_t before = carry;
    for (int k = 0; k < w; ++k) before += ws[k];
    if (i < nblk) colpre[(size_t)b * nblk + i] = before + x - v;
    __syncthreads();
    if (threadIdx.x == 255) carry = before + x;
    __syncthreads();
  }
  if (threadIdx.x == 0) total[b] = carry;
}

// base[b] = sum_{b' < b} total[b'] (one block; B <= 4096)
__global__ void __launch_bounds__(1024) k_part_base(const unsigned long long* __restrict__ total, uint32_t B,
                                                    unsigned long long* __restrict__ base) {
  __shared__ unsigned long long ws[32];
  __shared__ unsigned long long carry;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  for (uint32_t o0 = 0; o0 < B; o0 += 1024) {
    const uint32_t i = o0 + threadIdx.x;
    const unsigned long long v = i < B ? total[i] : 0;
    unsigned long long x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const unsigned long long y = __shfl_up_sync(kFull, x, o);
      if (lane >= o) x += y;
    }
    if (lane == 31) ws[w] = x;
    __syncthreads();
    unsigned long long before = carry;
    for (int k = 0; k < w; ++k) before += ws[k];
    if (i < B) base[i] = before + x - v;
    __syncthreads();
    if (threadIdx.x == 1023) carry = before + x;
    __syncthreads();
  }
}

// smem: cnt[8][B] (this round's tile counts per warp), pre[8][B] (exclusive over warps), run[B]
__global__ void __launch_bounds__(kPB) k_part_scatter(Chunk c, const uint8_t* __restrict__ stage,
                                                      const LaneDesc* __restrict__ lanes,
                                                      const uint64_t* __restrict__ tile_base, int bits,
                                                      const uint32_t* __restrict__ colpre,
                                                      const unsigned long long* __restrict__ base,
                                                      uint4* __restrict__ out) {
  extern __shared__ uint32_t sh[];
  const uint32_t B = 1u << bits;
  uint32_t* cnt = sh;                 // [8][B]
  uint32_t* run = sh + 8 * B;         // [B] records of this block already placed (earlier rounds)
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (uint32_t b = threadIdx.x; b < B; b += blockDim.x) run[b] = 0;
  uint32_t t0, t1;
  block_tiles(c.ntiles, gridDim.x, blockIdx.x, t0, t1);
  const uint32_t nblk = gridDim.x;
  for (uint32_t r0 = t0; r0 < t1; r0 += kPB / 32) {  // one round = up to 8 consecutive tiles
    const uint32_t ti = r0 + w;
    const bool have = ti < t1;
    for (uint32_t b = lane; b < B; b += 32) cnt[w * B + b] = 0;
    __syncwarp();
    LaneDesc d{0, 0, 0};
    if (have) d = lanes[(size_t)ti * 32 + lane];
    TileWalk tw;
    tw.init(d, lane);
    const uint8_t* tile = have ? stage + tile_base[ti] : nullptr;
    // pass 1: this tile's bucket counts
    for (uint32_t p0 = 0; p0 < tw.total; p0 += 32) {
      const uint32_t p = p0 + lane;
      int t;
      uint32_t j;
      tw.locate(p < tw.total ? p : tw.total - 1, t, j);
      if (p < tw.total) {
        const uint4 v = *reinterpret_cast<const uint4*>(tile + ((size_t)j * 32 + t) * 16);
        atomicAdd(&cnt[w * B + bucket_of((uint64_t)v.x | ((uint64_t)v.y << 32), bits)], 1u);
      }
    }
    __syncthreads();
    // exclusive prefix over the 8 tiles of this round, per bucket (in place), then advance run
    for (uint32_t b = threadIdx.x; b < B; b += blockDim.x) {
      uint32_t acc = run[b];
      for (int k = 0; k < kPB / 32; ++k) {
        const uint32_t x = cnt[k * B + b];
        cnt[k * B + b] = acc;
        acc += x;
      }
      run[b] = acc;
    }
    __syncthreads();
    // pass 2: ranks in record order, scatter
    for (uint32_t p0 = 0; p0 < tw.total; p0 += 32) {
      const uint32_t p = p0 + lane;
      const bool valid = p < tw.total;
      int t;
      uint32_t j;
      tw.locate(valid ? p : tw.total - 1, t, j);
      uint4 v = make_uint4(0, 0, 0, 0);
      uint32_t b = 0xffffffffu;
      if (valid) {
        v = *reinterpret_cast<const uint4*>(tile + ((size_t)j * 32 + t) * 16);
        b = bucket_of((uint64_t)v.x | ((uint64_t)v.y << 32), bits);
      }
      const unsigned m = __match_any_sync(kFull, b);
      const uint32_t rank = __popc(m & ((1u << lane) - 1));
      if (valid) {
        const unsigned long long pos = base[b] + colpre[(size_t)b * nblk + blockIdx.x] + cnt[w * B + b] + rank;
        out[pos] = v;
      }
      __syncwarp();
      if (valid && rank == 0) cnt[w * B + b] += __popc(m);   // leader advances this tile's bucket cursor
      __syncwarp();
    }
    __syncthreads();
  }
}

}  // namespace

size_t partition_smem(uint32_t B) { return (size_t)9 * B * 4; }

uint32_t partition_blocks(const Chunk& c) {
  uint32_t nblk = (c.ntiles + 7) / 8;
  if (nblk > (uint32_t)device_sms() * 2) nblk = (uint32_t)device_sms() * 2;
  return nblk ? nblk : 1;
}

void launch_partition(const Chunk& c, const uint8_t* stage, const LaneDesc* lanes, const uint64_t* tile_base,
                      int bits, uint32_t* hist, uint32_t* colpre, unsigned long long* total,
                      unsigned long long* base, uint8_t* out, cudaStream_t s) {
  const uint32_t B = 1u << bits, nblk = partition_blocks(c);
  k_part_hist<<<nblk, kPB, (size_t)B * 4, s>>>(c, stage, lanes, tile_base, bits, hist);
  k_part_cols<<<B, 256, 0, s>>>(hist, nblk, colpre, total);
  k_part_base<<<1, 1024, 0, s>>>(total, B, base);
  k_part_scatter<<<nblk, kPB, partition_smem(B), s>>>(c, stage, lanes, tile_base, bits, colpre, base,
                                                      reinterpret_cast<uint4*>(out));
}

cudaError_t configure_partition_kernels() {
  return cudaFuncSetAttribute(k_part_scatter, cudaFuncAttributeMaxDynamicSharedMemorySize, 9 * 4096 * 4);
}

}  // namespace bk
