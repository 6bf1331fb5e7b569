// kernels_pattern.cu — online pattern recognition of the address-generation stage (§IV.A,
// P:711-755; NEXT row f2 of SURVEY §8(f)). Each lane (thread) generates the element addresses its
// compute would touch — records in lane order, extents in access order, `elem` bytes per element
// (1 for text, 4 for fp32 fields) — keeps the first T in a private temporary buffer ("a few tens of
// bytes"), looks for the smallest period p <= pmax of address deltas confirmed by at
// least one delta past the first period, then verifies every later address against it ("verifies
// that each subsequently generated address follows the identified pattern"); the first
// mismatch falls back to explicit addresses. Per lane: p (0 = explicit), base, strides, count;
// totals give the Table II comparison: bytes of explicit addresses vs patterns.
#include "bk_internal.cuh"

namespace bk {
namespace {

constexpr int kTMax = 16, kPMax = 4;

struct PatternOut {
  int32_t* p;            // per lane: period, 0 = explicit addresses
  int64_t* strides;      // per lane: kPMax entries
  uint64_t* base;        // per lane: first address
  uint64_t* count;       // per lane: number of addresses
  unsigned long long* totals;  // [0] lanes, [1] pattern lanes, [2] addresses, [3] explicit addresses, [4] pattern bytes
};

__device__ __forceinline__ uint64_t rstart(const Chunk& c, const Access& a, const uint64_t* meta, uint64_t r) {
  if (a.rec_size) return r * a.rec_size;
  return r == c.hi ? c.end_byte : meta[r - c.lo];
}

__global__ void __launch_bounds__(256) k_addr_patterns(Chunk c, Access a, const uint64_t* __restrict__ meta,
                                                       const LaneDesc* __restrict__ lanes, uint32_t elem, uint32_t T,
                                                       uint32_t pmax, PatternOut o, int dump) {
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= c.L) return;
  const LaneDesc d = lanes[t];
  uint64_t buf[kTMax];
  int64_t st[kPMax];
  uint64_t n = 0, prev = 0, base = 0;
  int p = -1;          // -1: still filling the temp buffer; 0: explicit; >0: verified so far
  auto detect = [&](uint32_t m) -> int {  // smallest confirmed period over buf[0..m)
    if (m < 2) return 0;
    for (uint32_t q = 1; q <= pmax && q + 1 < m; ++q) {
      bool ok = true;
      for (uint32_t k = 0; k + 1 < m && ok; ++k)
        ok = (int64_t)(buf[k + 1] - buf[k]) == (int64_t)(buf[(k % q) + 1] - buf[k % q]);
      if (ok) {
        for (uint32_t z = 0; z < q; ++z) st[z] = (int64_t)(buf[z + 1] - buf[z]);
        return (int)q;
      }
    }
    return 0;
  };
  auto visit = [&](uint64_t addr) {
    if (n == 0) base = addr;
    if (p < 0) {
      buf[n] = addr;
      if (n + 1 == T) p = detect(T);
    } else if (p > 0) {
      if ((int64_t)(addr - prev) != st[(n - 1) % (uint64_t)p]) p = 0;  // mismatch: explicit from now on
    }
    prev = addr;
    ++n;
  };
  for (uint32_t j = 0; j < d.nrec; ++j) {
    const uint64_t r = d.first + j;
    const uint64_t rs = rstart(c, a, meta, r);
    const uint32_t ne = a.whole ? 1 : a.n_ext;
    for (uint32_t e = 0; e < ne; ++e) {
      const uint64_t xs = a.whole ? rs : rs + a.ext_off[e];
      const uint64_t xl = a.whole ? rstart(c, a, meta, r + 1) - rs : a.ext_len[e];
      for (uint64_t x = 0; x < xl; x += elem) visit(xs + x);
    }
  }
  if (p < 0) p = detect((uint32_t)n);   // fewer than T addresses in this lane
  if (dump) {
    o.p[t] = p;
    o.base[t] = base;
    o.count[t] = n;
    for (int z = 0; z < kPMax; ++z) o.strides[(size_t)t * kPMax + z] = z < p ? st[z] : 0;
  }
  atomicAdd(&o.totals[0], 1ull);
  atomicAdd(&o.totals[2], (unsigned long long)n);
  if (p > 0) {
    atomicAdd(&o.totals[1], 1ull);
    atomicAdd(&o.totals[4], 8ull + 8ull * (unsigned long long)p + 8ull);   // base + strides + count
  } else {
    atomicAdd(&o.totals[3], (unsigned long long)n);
  }
}

}  // namespace

void launch_addr_patterns(const Chunk& c, const Access& a, const uint64_t* meta, const LaneDesc* lanes, uint32_t elem,
                          uint32_t T, uint32_t pmax, int32_t* lane_p, int64_t* lane_strides, uint64_t* lane_base,
                          uint64_t* lane_count, unsigned long long* totals, int dump, cudaStream_t s) {
  PatternOut o{lane_p, lane_strides, lane_base, lane_count, totals};
  k_addr_patterns<<<(c.L + 255) / 256, 256, 0, s>>>(c, a, meta, lanes, elem, T, pmax, o, dump);
}

}  // namespace bk
