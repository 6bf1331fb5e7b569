// tma.cuh — bulk-copy (TMA engine) staging of warp tiles into shared memory, sm_100a.
//
// Stage 4 reads the chunk the way stage 2 laid it out: a warp tile is K rows of 512 B, row k
// holding word k of the tile's 32 lanes. A compute warp therefore needs its tile
// as one contiguous byte range, which is exactly what `cp.async.bulk` moves: one elected lane arms
// an mbarrier with the byte count and issues the copy; the copy engine writes shared memory and
// completes the transaction count; every lane waits on the barrier's phase, then reads its own
// 16-B word of each row from shared memory (conflict-free: 32 consecutive 16-B words).
//
// WarpTileStream walks the warp's tiles (w = first, first + stride, ...) in pieces of at most
// `rows` rows through two shared-memory buffers, so the copy of piece i+1 is in flight while the
// warp computes on piece i (north_star: "TMA or cp.async shared-memory staging of the
// interleaved chunk").
#pragma once
#include <stdint.h>

#include "bk_internal.cuh"

namespace bk {

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}

// make the initialised barriers visible to the async (copy-engine) proxy
__device__ __forceinline__ void mbar_fence_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}

// order this thread's earlier generic-proxy shared-memory accesses before later async-proxy writes
__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}

// global -> shared bulk copy; bytes % 16 == 0, both addresses 16-B aligned. The staged chunk is
// read exactly once, so the copy carries an L2 evict-first policy.
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  uint64_t pol;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol)
      : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred P1;\n"
      "LAB_WAIT:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
      "@P1 bra DONE;\n\t"
      "bra LAB_WAIT;\n"
      "DONE:\n\t}" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}

// Shared memory a WarpTileStream needs per warp: two buffers + two barriers.
__host__ __device__ constexpr size_t tile_stream_smem(uint32_t rows) { return 2ull * rows * 512 + 16; }

// One warp's double-buffered stream of (tile, piece) units over the tiles first, first+stride, ...
// `rows` (rows per piece) must be a multiple of the rows one record spans, so a record never
// straddles two pieces. All 32 lanes call every member; lane 0 issues the copies.
// kTma = false walks the same units but hands out the rows in place (HBM, plain 16-B loads): the
// variant for chunks that compute while zero-copy gathers are in flight, where bulk copies were
// measured to stall behind the SMs' outstanding sysmem reads (profiles/r01_tma.md).
template <bool kTma = true>
struct WarpTileStream {
  const uint8_t* stage;
  const uint64_t* tile_base;
  uint32_t ntiles, stride, rows;
  uint8_t* buf;    // 2 * rows * 512 B
  uint64_t* bar;   // 2 barriers
  // current unit
  uint32_t w, p, K;
  uint32_t b, phase;  // buffer of the current unit; per-buffer parity bits (bit b)

  __device__ __forceinline__ uint32_t tile_rows(uint32_t t) const {
    return (uint32_t)((tile_base[t + 1] - tile_base[t]) >> 9);
  }
  // next non-empty tile at or after t (stride steps), or ntiles
  __device__ __forceinline__ void seek(uint32_t& t, uint32_t& k) const {
    for (; t < ntiles; t += stride) {
      k = tile_rows(t);
      if (k) return;
    }
    k = 0;
  }
  __device__ __forceinline__ void issue(uint32_t t, uint32_t piece, uint32_t k, uint32_t buffer) {
    if (kTma && (threadIdx.x & 31) == 0) {
      const uint32_t r0 = piece * rows;
      const uint32_t n = (k - r0 < rows ? k - r0 : rows) * 512;
      fence_proxy_async_smem();
      mbar_arrive_expect_tx(bar + buffer, n);
      bulk_g2s(buf + (size_t)buffer * rows * 512, stage + tile_base[t] + (size_t)r0 * 512, n, bar + buffer);
    }
  }
  // Barriers are initialised by the caller (lane 0, count 1) before the block-wide sync.
  __device__ __forceinline__ void begin(uint32_t first) {
    w = first;
    p = 0;
    b = 0;
    phase = 0;
    seek(w, K);
    if (w < ntiles) issue(w, 0, K, 0);
  }
  __device__ __forceinline__ bool valid() const { return w < ntiles; }
  // Prefetch the next unit into the other buffer (its previous contents were consumed and the
  // warp synchronised at the end of the previous step), then wait for the current one.
  // Returns a pointer to the current piece's first row; rows [p*rows, min(K, (p+1)*rows)).
  __device__ __forceinline__ const uint8_t* acquire(uint32_t& nw, uint32_t& np, uint32_t& nK) {
    nw = w;
    np = p + 1;
    nK = K;
    if (np * rows >= K) {
      nw = w + stride;
      np = 0;
      seek(nw, nK);
    }
    if (!kTma) return stage + tile_base[w] + (size_t)p * rows * 512;
    if (nw < ntiles) issue(nw, np, nK, b ^ 1);
    mbar_wait(bar + b, (phase >> b) & 1);
    phase ^= 1u << b;
    return buf + (size_t)b * rows * 512;
  }
  __device__ __forceinline__ void release(uint32_t nw, uint32_t np, uint32_t nK) {
    if (kTma) __syncwarp();
    w = nw;
    p = np;
    K = nK;
    b ^= 1;
  }
};

// Shared memory of `nwarp` warp streams (buffers, then barriers); none without TMA.
template <bool kTma>
__host__ __device__ constexpr size_t stream_smem(uint32_t nwarp, uint32_t rows) {
  return kTma ? nwarp * tile_stream_smem(rows) : 0;
}

// This warp's stream over the tiles of a chunk, its buffers and barriers carved from `smem`
// (layout of stream_smem); lane 0 initialises the barriers. Call with the whole warp.
template <bool kTma>
__device__ __forceinline__ WarpTileStream<kTma> warp_stream(unsigned char* smem, uint32_t nwarp, uint32_t rows,
                                                            const uint8_t* stage, const uint64_t* tile_base,
                                                            uint32_t ntiles) {
  const uint32_t wid = threadIdx.x >> 5;
  WarpTileStream<kTma> ts{};
  ts.stage = stage;
  ts.tile_base = tile_base;
  ts.ntiles = ntiles;
  ts.stride = gridDim.x * nwarp;
  ts.rows = rows;
  if (kTma) {
    ts.buf = smem + (size_t)wid * 2 * rows * 512;
    ts.bar = reinterpret_cast<uint64_t*>(smem + (size_t)nwarp * 2 * rows * 512) + 2 * wid;
    if ((threadIdx.x & 31) == 0) {
      mbar_init(ts.bar, 1);
      mbar_init(ts.bar + 1, 1);
      mbar_fence_init();
    }
    __syncwarp();
  }
  return ts;
}

}  // namespace bk
