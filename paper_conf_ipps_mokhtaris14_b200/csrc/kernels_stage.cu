// kernels_stage.cu — pipeline stages 1 and 2 (+3 in zero-copy mode) for sm_100a.
//
// Stage 1, address generation (Fig. 3): instead of
// recording one address per access (addrBuf[counter][tid]) the GPU emits one compact lane
// descriptor per thread {first record, record count, accessed bytes} — the statically known
// pattern of a hand-written kernel (P:711-755 pattern recognition) — plus the
// warp-tile sizes and their exclusive scan (tile bases).
//
// Stage 2, assembly: gather exactly the accessed bytes into warp tiles
// where word k of lane t sits at tile_base(t/32) + (k*32 + t%32)*16, i.e. the paper's
// buf[counter][tid] layout with 16-byte elements, so that 32 lanes reading their k-th word
// issue one 512-byte coalesced access. When `src` is pinned, mapped host memory the gather
// kernel is also stage 3 (the transfer): it pulls the bytes over PCIe with 16-byte loads.
#include "bk_internal.cuh"

#include <algorithm>

namespace bk {
namespace {

constexpr unsigned kFull = 0xffffffffu;

__device__ __forceinline__ uint64_t rec_off(const Chunk& c, const Access& a, const uint64_t* meta, uint64_t r) {
  if (a.rec_size) return r * a.rec_size;
  return r == c.hi ? c.end_byte : meta[r - c.lo];
}

// A(lo, r): accessed bytes of records [lo, r).
__device__ __forceinline__ uint64_t acc_bytes(const Chunk& c, const Access& a, const uint64_t* meta, uint64_t r) {
  if (!a.whole) return (r - c.lo) * a.E;
  if (a.rec_size) return (r - c.lo) * a.rec_size;
  return rec_off(c, a, meta, r) - c.base_byte;
}

// first(t) = min{ r in [lo,hi] : A(lo,r) >= floor(t*A(lo,hi)/L) }, first(L) = hi.
__device__ __forceinline__ uint64_t lane_first(const Chunk& c, const Access& a, const uint64_t* meta, uint32_t t) {
  if (t >= c.L) return c.hi;
  const uint64_t target = (uint64_t)t * c.accessed / c.L;  // host guarantees no overflow
  uint64_t per = a.whole ? a.rec_size : a.E;
  if (a.whole && a.rec_size == 0) {
    uint64_t lo = c.lo, hi = c.hi;
    while (lo < hi) {
      uint64_t mid = lo + (hi - lo) / 2;
      if (acc_bytes(c, a, meta, mid) >= target) hi = mid; else lo = mid + 1;
    }
    return lo;
  }
  if (per == 0) return c.lo;
  uint64_t k = (target + per - 1) / per;
  return c.lo + k < c.hi ? c.lo + k : c.hi;
}

// Whole variable-length records: the same rule evaluated from the records' side, so no lane
// needs a binary search (a chain of ~log2(n) dependent loads). With A_j = A(lo, lo+j),
//   first(t) = lo+j  <=>  A_{j-1} < floor(t*A/L) <= A_j  <=>  ceil((A_{j-1}+1)L/A) <= t < ceil((A_j+1)L/A)
// (j = 0: from t = 0). One thread per record boundary j in [0, n] writes lanes[t].first for its t
// range. `src` holds off[lo..hi-1] (HBM, or the registered offsets read zero-copy, in which case
// they are also copied to `meta_out` for the later stages).
__global__ void __launch_bounds__(256) k_lane_first(Chunk c, const uint64_t* __restrict__ src,
                                                    uint64_t* __restrict__ meta_out, LaneDesc* __restrict__ lanes) {
  const uint64_t n = c.hi - c.lo;
  const uint64_t j = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  const int lane = threadIdx.x & 31;
  uint64_t Aj = 0;
  if (j < n) {
    const uint64_t o = __ldcs(src + j);
    if (meta_out) meta_out[j] = o;
    Aj = o - c.base_byte;
  } else if (j == n) {
    Aj = c.end_byte - c.base_byte;
  }
  uint64_t Ap = __shfl_up_sync(kFull, Aj, 1);
  if (lane == 0 && j > 0 && j <= n) Ap = __ldcs(src + j - 1) - c.base_byte;
  if (j > n) return;
  const uint64_t A = c.accessed, L = c.L;
  uint64_t t0, t1;
  if (A == 0) {
    t0 = 0;
    t1 = j == 0 ? L : 0;
  } else {
    t0 = j == 0 ? 0 : ((Ap + 1) * L + A - 1) / A;
    t1 = ((Aj + 1) * L + A - 1) / A;
    if (t1 > L) t1 = L;
  }
  for (uint64_t t = t0; t < t1; ++t) lanes[t].first = c.lo + j;
}

template <bool kPre>  // kPre: lanes[].first already written by k_lane_first
__global__ void __launch_bounds__(256) k_addrgen(Chunk c, Access a, const uint64_t* __restrict__ meta,
                                                 LaneDesc* __restrict__ lanes, uint32_t* __restrict__ tileK) {
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= c.L) return;  // L % 32 == 0: whole warps leave together
  uint64_t f0, f1;
  if (kPre) {
    f0 = lanes[t].first;
    f1 = t + 1 < c.L ? lanes[t + 1].first : c.hi;
  } else {
    f0 = lane_first(c, a, meta, t);
    f1 = lane_first(c, a, meta, t + 1);
  }
  const uint64_t nb = acc_bytes(c, a, meta, f1) - acc_bytes(c, a, meta, f0);
  if (kPre) {  // leave .first alone: the neighbouring lane reads it
    *reinterpret_cast<uint2*>(&lanes[t].nrec) = make_uint2((uint32_t)(f1 - f0), (uint32_t)nb);
  } else {
    LaneDesc d;
    d.first = f0;
    d.nrec = (uint32_t)(f1 - f0);
    d.nbytes = (uint32_t)nb;
    lanes[t] = d;
  }
  const uint32_t K = __reduce_max_sync(kFull, (uint32_t)((nb + 15) >> 4));
  if ((t & 31) == 0) tileK[t >> 5] = K;
}

// tile_base[w] = 512 * sum_{w' < w} K_w'; tile_base[ntiles] = staged size.
__global__ void __launch_bounds__(1024) k_tile_scan(const uint32_t* __restrict__ tileK, uint32_t ntiles,
                                                    uint64_t* __restrict__ tile_base, uint64_t cap, int* err,
                                                    unsigned long long* staged_sum) {
  __shared__ uint64_t warp_sums[32];
  __shared__ uint64_t carry;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  for (uint32_t base = 0; base < ntiles; base += 1024) {
    const uint32_t i = base + threadIdx.x;
    uint64_t v = i < ntiles ? 512ull * tileK[i] : 0;
    uint64_t x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      uint64_t y = __shfl_up_sync(kFull, x, o);
      if (lane >= o) x += y;
    }
    if (lane == 31) warp_sums[wid] = x;
    __syncthreads();
    if (wid == 0) {
      uint64_t s = warp_sums[lane];
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        uint64_t y = __shfl_up_sync(kFull, s, o);
        if (lane >= o) s += y;
      }
      warp_sums[lane] = s;
    }
    __syncthreads();
    const uint64_t excl = carry + (wid ? warp_sums[wid - 1] : 0) + x - v;
    if (i < ntiles) tile_base[i] = excl;
    __syncthreads();
    if (threadIdx.x == 1023) carry = excl + v;
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    tile_base[ntiles] = carry;
    atomicAdd(staged_sum, (unsigned long long)carry);
    if (carry > cap) atomicOr(err, kErrStageOverflow);
  }
}

template <bool kHost>
__device__ __forceinline__ uint4 ld16(const uint4* p) {
  if (kHost) return __ldcs(p);   // streaming: host bytes are read exactly once
  return __ldcs(p);
}

// 16-B aligned load limited to the readable source range [lo, hi): interior words are one vector
// load; a word straddling a bound (data-set edges only) is assembled from in-range bytes.
template <bool kHost>
__device__ __forceinline__ uint4 ld16b(const uint4* p, const uint8_t* lo, const uint8_t* hi) {
  const uint8_t* b = reinterpret_cast<const uint8_t*>(p);
  if (b >= lo && b + 16 <= hi) return ld16<kHost>(p);
  uint32_t w[4] = {0, 0, 0, 0};
  for (int q = 0; q < 16; ++q)
    if (b + q >= lo && b + q < hi) w[q >> 2] |= (uint32_t)b[q] << (8 * (q & 3));
  return make_uint4(w[0], w[1], w[2], w[3]);
}

// out bytes q = concat(a, b)[s + q], s in [0, 16)
__device__ __forceinline__ uint4 shift_bytes(uint4 a, uint4 b, uint32_t s) {
  const uint32_t bs = (s & 3) * 8;
  uint32_t w0, w1, w2, w3, w4;
  switch (s >> 2) {
    case 0: w0 = a.x; w1 = a.y; w2 = a.z; w3 = a.w; w4 = b.x; break;
    case 1: w0 = a.y; w1 = a.z; w2 = a.w; w3 = b.x; w4 = b.y; break;
    case 2: w0 = a.z; w1 = a.w; w2 = b.x; w3 = b.y; w4 = b.z; break;
    default: w0 = a.w; w1 = b.x; w2 = b.y; w3 = b.z; w4 = b.w; break;
  }
  uint4 o;
  o.x = __funnelshift_r(w0, w1, bs);
  o.y = __funnelshift_r(w1, w2, bs);
  o.z = __funnelshift_r(w2, w3, bs);
  o.w = __funnelshift_r(w3, w4, bs);
  return o;
}

// keep the first `valid` bytes (valid < 16), zero the rest
__device__ __forceinline__ uint4 keep_bytes(uint4 v, uint32_t valid) {
  uint32_t w[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    int keep = (int)valid - 4 * i;
    uint32_t m = keep >= 4 ? 0xffffffffu : keep <= 0 ? 0u : (0xffffffffu >> (32 - 8 * keep));
    w[i] &= m;
  }
  return make_uint4(w[0], w[1], w[2], w[3]);
}

__device__ __forceinline__ uint4 shfl_u4(uint4 v, int src, int width = 32) {
  return make_uint4(__shfl_sync(kFull, v.x, src, width), __shfl_sync(kFull, v.y, src, width),
                    __shfl_sync(kFull, v.z, src, width), __shfl_sync(kFull, v.w, src, width));
}
__device__ __forceinline__ uint4 shfl_down_u4(uint4 v, int d, int width = 32) {
  return make_uint4(__shfl_down_sync(kFull, v.x, d, width), __shfl_down_sync(kFull, v.y, d, width),
                    __shfl_down_sync(kFull, v.z, d, width), __shfl_down_sync(kFull, v.w, d, width));
}

__device__ __forceinline__ void zero_holes(uint8_t* tile, uint32_t K, uint32_t W, int lane) {
  for (uint32_t k = W; k < K; ++k)
    *reinterpret_cast<uint4*>(tile + ((size_t)k * 32 + lane) * 16) = make_uint4(0, 0, 0, 0);
}

// WHOLE-record access: a tile's 32 lanes cover one contiguous byte range, so one warp streams
// it with coalesced 16-B loads (each source byte read once; 512 B per warp load) and routes
// each aligned input word to the lane/word it starts, shifting by that lane's misalignment.
template <bool kHost>
__global__ void __launch_bounds__(256) k_gather_whole(Chunk c, Access a, const uint8_t* __restrict__ src,
                                                      const uint64_t* __restrict__ meta,
                                                      const LaneDesc* __restrict__ lanes,
                                                      const uint64_t* __restrict__ tile_base,
                                                      uint8_t* __restrict__ stage, uint64_t cap, uint32_t U) {
  if (tile_base[c.ntiles] > cap) return;  // stage-1 flagged an overflow: never write past the slot
  const uint8_t* glo = src - c.guard_lo;
  const uint8_t* ghi = src + c.guard_hi;
  const int lane = threadIdx.x & 31;
  const uint32_t nw_grid = gridDim.x * (blockDim.x >> 5);
  // U warps per tile: warp u streams the tile's 512-B blocks [u*NB/U, (u+1)*NB/U), so a chunk
  // with few tiles still spreads its loads over every SM.
  for (uint32_t vw = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); vw < c.ntiles * U; vw += nw_grid) {
    const uint32_t w = vw / U, u = vw % U;
    const LaneDesc d = lanes[(size_t)w * 32 + lane];
    const uint64_t rel = rec_off(c, a, meta, d.first) - c.base_byte;
    const uint64_t rel0 = __shfl_sync(kFull, rel, 0);
    const uintptr_t abase = (uintptr_t)(src + rel0) & ~(uintptr_t)15;
    const uint64_t b = (uint64_t)((uintptr_t)(src + rel) - abase);  // lane start vs aligned stream
    const uint32_t sw = (uint32_t)(b >> 4), s = (uint32_t)(b & 15);
    const uint32_t W = (d.nbytes + 15) >> 4;
    const uint32_t ew = sw + W;
    const uint64_t bend = __shfl_sync(kFull, b + d.nbytes, 31);
    const uint32_t NW = (uint32_t)((bend + 15) >> 4);
    uint8_t* tile = stage + tile_base[w];
    const uint32_t K = (uint32_t)((tile_base[w + 1] - tile_base[w]) >> 9);
    const uint4* in = reinterpret_cast<const uint4*>(abase);
    // kDepth 512-B warp loads in flight per warp (PCIe latency x bandwidth needs ~100 KB in
    // flight chip-wide; a chunk may have only a few hundred tiles)
    constexpr int kDepth = 4;
    const uint32_t NB = (NW + 31) >> 5;
    const uint32_t b0 = (uint32_t)((uint64_t)u * NB / U), b1 = (uint32_t)((uint64_t)(u + 1) * NB / U);
    const uint32_t jend = min(NW, b1 * 32);  // words of this warp's range
    uint4 ring[kDepth];
#pragma unroll
    for (int i = 0; i < kDepth; ++i) {
      const uint32_t jj = (b0 + i) * 32 + lane;
      ring[i] = jj < jend ? ld16b<kHost>(in + jj, glo, ghi) : make_uint4(0, 0, 0, 0);
    }
    // the word after the range: the high half of lane 31's shift window in the last block
    const uint4 extra = (lane == 0 && b1 > b0 && b1 * 32 < NW) ? ld16b<kHost>(in + b1 * 32, glo, ghi)
                                                              : make_uint4(0, 0, 0, 0);
    for (uint32_t blk = b0; blk < b1; ++blk) {
      const uint4 cur = ring[0];
      uint4 hi = shfl_down_u4(cur, 1);
      const uint4 n0 = shfl_u4(blk + 1 < b1 ? ring[1] : extra, 0);
      if (lane == 31) hi = n0;
#pragma unroll
      for (int i = 0; i + 1 < kDepth; ++i) ring[i] = ring[i + 1];
      {
        const uint32_t jn = (blk + kDepth) * 32 + lane;
        ring[kDepth - 1] = jn < jend ? ld16b<kHost>(in + jn, glo, ghi) : make_uint4(0, 0, 0, 0);
      }
      const uint32_t j = blk * 32 + lane;
      // ta = last lane whose first word is <= j (sw is non-decreasing over lanes)
      int ta = 0;
#pragma unroll
      for (int step = 16; step; step >>= 1) {
        const uint32_t v = __shfl_sync(kFull, sw, ta + step);
        if (v <= j) ta += step;
      }
      int t = ta;
      bool active = j < NW;
      while (__any_sync(kFull, active)) {
        const int tt = active ? t : 0;
        const uint32_t swt = __shfl_sync(kFull, sw, tt);
        const uint32_t ewt = __shfl_sync(kFull, ew, tt);
        const uint32_t st = __shfl_sync(kFull, s, tt);
        const uint32_t nbt = __shfl_sync(kFull, d.nbytes, tt);
        if (active) {
          if (swt <= j && j < ewt) {
            const uint32_t k = j - swt;
            uint4 o = shift_bytes(cur, hi, st);
            const uint32_t valid = nbt - 16 * k;
            if (valid < 16) o = keep_bytes(o, valid);
            *reinterpret_cast<uint4*>(tile + ((size_t)k * 32 + tt) * 16) = o;
          }
          if (swt == j && tt > 0) t = tt - 1; else active = false;
        }
      }
    }
    if (u == 0) zero_holes(tile, K, W, lane);
  }
}

// Fixed extents per record, single extent of E = 16*EW bytes: a group of G >= EW+1 threads
// copies one record's extent (the group's 16-B loads of one record coalesce into one request
// per 128-B line), shifts it into place and writes words k = j*EW .. j*EW+EW-1 of lane t.
template <bool kHost, int G>
__global__ void __launch_bounds__(256) k_gather_field(Chunk c, Access a, const uint8_t* __restrict__ src,
                                                      const uint64_t* __restrict__ meta,
                                                      const LaneDesc* __restrict__ lanes,
                                                      const uint64_t* __restrict__ tile_base,
                                                      uint8_t* __restrict__ stage, uint64_t cap) {
  if (tile_base[c.ntiles] > cap) return;  // stage-1 flagged an overflow: never write past the slot
  const uint8_t* glo = src - c.guard_lo;
  const uint8_t* ghi = src + c.guard_hi;
  const int lane = threadIdx.x & 31;
  const int g = lane / G, q = lane % G;
  const uint32_t EW = a.E >> 4;
  const uint32_t eo = a.ext_off[0];
  const uint32_t nw_grid = gridDim.x * (blockDim.x >> 5);
  for (uint32_t w = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); w < c.ntiles; w += nw_grid) {
    const LaneDesc d = lanes[(size_t)w * 32 + lane];
    uint32_t incl = d.nrec;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(kFull, incl, o);
      if (lane >= o) incl += y;
    }
    const uint32_t total = __shfl_sync(kFull, incl, 31);
    uint8_t* tile = stage + tile_base[w];
    const uint32_t K = (uint32_t)((tile_base[w + 1] - tile_base[w]) >> 9);
    for (uint32_t base = 0; base < total; base += 32 / G) {
      const uint32_t job = base + g;
      const bool valid = job < total;
      // t = number of lanes with incl <= job
      int t = 0;
#pragma unroll
      for (int step = 16; step; step >>= 1) {
        const uint32_t v = __shfl_sync(kFull, incl, t + step - 1);
        if (v <= job) t += step;
      }
      t = t > 31 ? 31 : t;
      const uint32_t incl_t = __shfl_sync(kFull, incl, t);
      const uint32_t nrec_t = __shfl_sync(kFull, d.nrec, t);
      const uint64_t first_t = __shfl_sync(kFull, d.first, t);
      const uint32_t j = job - (incl_t - nrec_t);
      const uint64_t r = first_t + j;
      uint4 v = make_uint4(0, 0, 0, 0);
      uint32_t s = 0;
      if (valid) {
        const uint8_t* p = src + (rec_off(c, a, meta, r) - c.base_byte) + eo;
        const uintptr_t ab = (uintptr_t)p & ~(uintptr_t)15;
        s = (uint32_t)((uintptr_t)p - ab);
        const uint32_t NI = (s + a.E + 15) >> 4;
        if ((uint32_t)q < NI) v = ld16b<kHost>(reinterpret_cast<const uint4*>(ab) + q, glo, ghi);
      }
      const uint4 hi = shfl_down_u4(v, 1, G);
      if (valid && (uint32_t)q < EW) {
        const uint4 o = shift_bytes(v, hi, s);
        *reinterpret_cast<uint4*>(tile + ((size_t)(j * EW + q) * 32 + t) * 16) = o;
      }
    }
    zero_holes(tile, K, (d.nbytes + 15) >> 4, lane);
  }
}

// Any extent list (multi-extent, unaligned lengths, duplicates): one thread per record,
// byte by byte. Correct for every spec; used only where no fast path applies.
template <bool kHost>
__global__ void __launch_bounds__(256) k_gather_bytes(Chunk c, Access a, const uint8_t* __restrict__ src,
                                                      const uint64_t* __restrict__ meta,
                                                      const LaneDesc* __restrict__ lanes,
                                                      const uint64_t* __restrict__ tile_base,
                                                      uint8_t* __restrict__ stage, uint64_t cap) {
  if (tile_base[c.ntiles] > cap) return;  // stage-1 flagged an overflow: never write past the slot
  const uint8_t* glo = src - c.guard_lo;
  const uint8_t* ghi = src + c.guard_hi;
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= c.L) return;
  const int lane = t & 31;
  const uint32_t w = t >> 5;
  const LaneDesc d = lanes[t];
  uint8_t* tile = stage + tile_base[w];
  const uint32_t K = (uint32_t)((tile_base[w + 1] - tile_base[w]) >> 9);
  uint64_t b = 0;
  for (uint32_t j = 0; j < d.nrec; ++j) {
    const uint64_t r = d.first + j;
    const uint64_t rs = rec_off(c, a, meta, r) - c.base_byte;
    const uint32_t ne = a.whole ? 1 : a.n_ext;
    for (uint32_t e = 0; e < ne; ++e) {
      const uint64_t xs = a.whole ? rs : rs + a.ext_off[e];
      const uint64_t xl = a.whole ? rec_off(c, a, meta, r + 1) - c.base_byte - rs : a.ext_len[e];
      for (uint64_t x = 0; x < xl; ++x, ++b)
        tile[((b >> 4) * 32 + lane) * 16 + (b & 15)] = src[xs + x];
    }
  }
  // zero the tail of the last word and the holes
  for (; b & 15; ++b) tile[((b >> 4) * 32 + lane) * 16 + (b & 15)] = 0;
  for (uint32_t k = (uint32_t)(b >> 4); k < K; ++k)
    *reinterpret_cast<uint4*>(tile + ((size_t)k * 32 + lane) * 16) = make_uint4(0, 0, 0, 0);
}

}  // namespace

__global__ void k_spin(long long cycles) {
  const long long t0 = clock64();
  while (clock64() - t0 < cycles) {
  }
}

void launch_spin(long long cycles, cudaStream_t s) { k_spin<<<1, 1, 0, s>>>(cycles); }

void launch_addrgen(const Chunk& c, const Access& a, const uint64_t* meta, LaneDesc* lanes, uint32_t* tileK,
                    uint64_t* tile_base, uint64_t stage_cap, int* err, unsigned long long* staged_sum,
                    cudaStream_t s, const uint64_t* meta_src) {
  if (a.whole && a.rec_size == 0) {
    const uint64_t nb = c.hi - c.lo + 1;
    k_lane_first<<<(uint32_t)((nb + 255) / 256), 256, 0, s>>>(c, meta_src ? meta_src : meta,
                                                               meta_src ? const_cast<uint64_t*>(meta) : nullptr, lanes);
    k_addrgen<true><<<(c.L + 255) / 256, 256, 0, s>>>(c, a, meta, lanes, tileK);
  } else {
    k_addrgen<false><<<(c.L + 255) / 256, 256, 0, s>>>(c, a, meta, lanes, tileK);
  }
  k_tile_scan<<<1, 1024, 0, s>>>(tileK, c.ntiles, tile_base, stage_cap, err, staged_sum);
}

void launch_tile_scan(const uint32_t* tileK, uint32_t ntiles, uint64_t* tile_base, uint64_t stage_cap, int* err,
                      unsigned long long* staged_sum, cudaStream_t s) {
  k_tile_scan<<<1, 1024, 0, s>>>(tileK, ntiles, tile_base, stage_cap, err, staged_sum);
}

template <bool kHost>
static void gather_impl(const Chunk& c, const Access& a, const uint8_t* src, const uint64_t* meta,
                        const LaneDesc* lanes, const uint64_t* tile_base, uint8_t* stage, uint64_t cap,
                        cudaStream_t s) {
  const uint32_t warps = c.ntiles;
  uint32_t grid = (warps + 7) / 8;
  // Zero-copy reads are bound by outstanding PCIe read requests (~1k tags), not by warps: one
  // block per SM keeps >1k 16-B requests in flight and leaves the other SMs' slots to the compute
  // kernels of earlier chunks running concurrently. HBM re-layout uses the whole chip.
  const uint32_t grid_cap = kHost ? (uint32_t)device_sms() : (uint32_t)device_sms() * 8;
  if (grid > grid_cap) grid = grid_cap;
  if (grid == 0) return;
  if (a.whole) {
    // split tiles over up to 8 warps until the chunk fills the grid cap's warps
    const uint32_t U = (uint32_t)std::min<uint64_t>(8, std::max<uint64_t>(1, (8ull * grid_cap + warps - 1) / warps));
    uint64_t g2 = ((uint64_t)warps * U + 7) / 8;
    k_gather_whole<kHost><<<(uint32_t)std::min<uint64_t>(g2, grid_cap), 256, 0, s>>>(c, a, src, meta, lanes,
                                                                                       tile_base, stage, cap, U);
    return;
  }
  const bool fast = a.n_ext == 1 && (a.E & 15) == 0 && a.E > 0;
  const uint32_t EW = a.E >> 4;
  if (fast && EW + 1 <= 2) { k_gather_field<kHost, 2><<<grid, 256, 0, s>>>(c, a, src, meta, lanes, tile_base, stage, cap); return; }
  if (fast && EW + 1 <= 4) { k_gather_field<kHost, 4><<<grid, 256, 0, s>>>(c, a, src, meta, lanes, tile_base, stage, cap); return; }
  if (fast && EW + 1 <= 8) { k_gather_field<kHost, 8><<<grid, 256, 0, s>>>(c, a, src, meta, lanes, tile_base, stage, cap); return; }
  if (fast && EW + 1 <= 16) { k_gather_field<kHost, 16><<<grid, 256, 0, s>>>(c, a, src, meta, lanes, tile_base, stage, cap); return; }
  if (fast && EW + 1 <= 32) { k_gather_field<kHost, 32><<<grid, 256, 0, s>>>(c, a, src, meta, lanes, tile_base, stage, cap); return; }
  k_gather_bytes<kHost><<<(c.L + 255) / 256, 256, 0, s>>>(c, a, src, meta, lanes, tile_base, stage, cap);
}

void launch_gather(const Chunk& c, const Access& a, const uint8_t* src, const uint64_t* meta, const LaneDesc* lanes,
                   const uint64_t* tile_base, uint8_t* stage, uint64_t cap, int zero_copy, cudaStream_t s) {
  if (zero_copy) gather_impl<true>(c, a, src, meta, lanes, tile_base, stage, cap, s);
  else gather_impl<false>(c, a, src, meta, lanes, tile_base, stage, cap, s);
}

}  // namespace bk
