// kernels_addr.cu — stage 1 in the paper's ADDRESS MODE (BK_GATHER_ADDR; §III P:244-255,
// P:376-394, Fig. 3, and §IV.A pattern recognition P:711-755): every lane (thread) generates
// the address of each element its compute will read, in access order, keeps the first T in a private
// temporary buffer, looks for a base + period-p stride pattern (p <= 4, confirmed by at least one
// delta past the first period), verifies every later address against it, and on the first mismatch
// "starts again without attempting to identify a pattern, writing the addresses to the CPU-side
// address buffer". What reaches the host (pinned, mapped memory, the paper's addrBuf):
// one 48-B descriptor per lane — the pattern, or "explicit" — plus the explicit lanes' addresses,
// compacted. The host then assembles the lanes' bytes (host_gather.cpp host_assemble_addr)
// and DMAs them; stage 4 is unchanged.
//
// Addresses are byte offsets into the registered data set; an element is `elem` bytes read at an
// address. Addresses come either from the access spec (built-in kernels: every extent of every
// record of the lane, elem-sized steps) or from a caller's generator kernel (bk_run_user_addr), which
// wrote each lane's addresses at user_addr[user_base[t] + k], k < user_count[t].
#include "bk_internal.cuh"

namespace bk {
namespace {

constexpr int kTMax = 16, kPMax = 4;

__device__ __forceinline__ uint64_t rstart(const Chunk& c, const Access& a, const uint64_t* meta, uint64_t r) {
  if (a.rec_size) return r * a.rec_size;
  return r == c.hi ? c.end_byte : meta[r - c.lo];
}

// Calls f(addr) for every element address of lane d under the access spec, in access order.
template <class F>
__device__ __forceinline__ void spec_addresses(const Chunk& c, const Access& a, const uint64_t* meta,
                                               const LaneDesc& d, uint32_t elem, F&& f) {
  for (uint32_t j = 0; j < d.nrec; ++j) {
    const uint64_t r = d.first + j;
    const uint64_t rs = rstart(c, a, meta, r);
    const uint32_t ne = a.whole ? 1 : a.n_ext;
    for (uint32_t e = 0; e < ne; ++e) {
      const uint64_t xs = a.whole ? rs : rs + a.ext_off[e];
      const uint64_t xl = a.whole ? rstart(c, a, meta, r + 1) - rs : a.ext_len[e];
      for (uint64_t x = 0; x < xl; x += elem) f(xs + x);
    }
  }
}

struct AddrSrc {              // where a lane's addresses come from
  const uint64_t* user_addr;  // nullptr: the access spec
  const uint64_t* user_base;
  const uint32_t* user_count;
};

template <class F>
__device__ __forceinline__ void lane_addresses(const Chunk& c, const Access& a, const uint64_t* meta,
                                               const LaneDesc& d, uint32_t t, uint32_t elem, const AddrSrc& src,
                                               F&& f) {
  if (src.user_addr) {
    const uint64_t b = src.user_base[t];
    const uint32_t cap = (uint32_t)(src.user_base[t + 1] - b);
    const uint32_t n = min(src.user_count[t], cap);   // a count above the capacity is cut here and
    for (uint32_t k = 0; k < n; ++k) f(src.user_addr[b + k]);   // reported by k_addr_detect
  } else {
    spec_addresses(c, a, meta, d, elem, f);
  }
}

// Detect / verify per lane; descriptor to the host, explicit count to ecount. User mode also sets the
// lane's staged size (count x elem) and its tile's word count for the tile scan.
__global__ void __launch_bounds__(256) k_addr_detect(Chunk c, Access a, const uint64_t* __restrict__ meta,
                                                     LaneDesc* __restrict__ lanes, uint32_t* __restrict__ tileK,
                                                     uint32_t elem, uint32_t T, uint32_t pmax, int patterns,
                                                     AddrSrc src, AddrDesc* __restrict__ desc,
                                                     uint32_t* __restrict__ ecount) {
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= c.L) return;   // L % 32 == 0: whole warps leave together
  const LaneDesc d = lanes[t];
  uint64_t buf[kTMax];
  int64_t st[kPMax] = {0, 0, 0, 0};
  uint64_t n = 0, prev = 0, base = 0;
  int p = patterns ? -1 : 0;   // -1: filling the temp buffer; 0: explicit; > 0: verified so far
  auto detect = [&](uint32_t m) -> int {   // smallest confirmed period over buf[0..m)
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
  lane_addresses(c, a, meta, d, t, elem, src, [&](uint64_t addr) {
    if (n == 0) base = addr;
    if (p < 0) {
      buf[n] = addr;
      if (n + 1 == T) p = detect(T);
    } else if (p > 0) {
      if ((int64_t)(addr - prev) != st[(n - 1) % (uint64_t)p]) p = 0;   // mismatch: explicit from now on
    }
    prev = addr;
    ++n;
  });
  if (p < 0) p = detect((uint32_t)n);   // fewer than T addresses in this lane
  AddrDesc o;
  o.base = base;
  for (int z = 0; z < kPMax; ++z) o.stride[z] = z < p ? st[z] : 0;
  o.count = (uint32_t)n;
  o.p = p;
  if (src.user_addr && src.user_count[t] > src.user_base[t + 1] - src.user_base[t])
    o.count = 0xffffffffu;   // over the lane's capacity: the host reports BK_E_INVAL
  desc[t] = o;
  ecount[t] = p > 0 ? 0u : (uint32_t)n;
  if (src.user_addr) {
    const uint32_t nb = (uint32_t)(n * elem);
    lanes[t].nbytes = nb;
    const uint32_t K = __reduce_max_sync(0xffffffffu, (nb + 15) >> 4);
    if ((t & 31) == 0) tileK[t >> 5] = K;
  }
}

// exclusive scan of the explicit counts (one block): epos[t], epos[L] = total
__global__ void __launch_bounds__(1024) k_addr_scan(const uint32_t* __restrict__ cnt, uint32_t L,
                                                    uint64_t* __restrict__ epos, uint64_t* __restrict__ total_host) {
  __shared__ uint64_t warp_sums[32];
  __shared__ uint64_t carry;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  for (uint32_t b = 0; b < L; b += 1024) {
    const uint32_t i = b + threadIdx.x;
    const uint64_t v = i < L ? cnt[i] : 0;
    uint64_t x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint64_t y = __shfl_up_sync(0xffffffffu, x, o);
      if (lane >= o) x += y;
    }
    if (lane == 31) warp_sums[wid] = x;
    __syncthreads();
    if (wid == 0) {
      uint64_t s = warp_sums[lane];
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint64_t y = __shfl_up_sync(0xffffffffu, s, o);
        if (lane >= o) s += y;
      }
      warp_sums[lane] = s;
    }
    __syncthreads();
    const uint64_t excl = carry + (wid ? warp_sums[wid - 1] : 0) + x - v;
    if (i < L) epos[i] = excl;
    __syncthreads();
    if (threadIdx.x == 1023) carry = excl + v;
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    epos[L] = carry;
    *total_host = carry;
  }
}

// explicit lanes: the addresses again, now written ("started again ... writing the addresses")
__global__ void __launch_bounds__(256) k_addr_emit(Chunk c, Access a, const uint64_t* __restrict__ meta,
                                                   const LaneDesc* __restrict__ lanes, uint32_t elem, AddrSrc src,
                                                   const uint32_t* __restrict__ ecount,
                                                   const uint64_t* __restrict__ epos, uint64_t* __restrict__ exp) {
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= c.L || ecount[t] == 0) return;
  uint64_t* o = exp + epos[t];
  uint64_t k = 0;
  lane_addresses(c, a, meta, lanes[t], t, elem, src, [&](uint64_t addr) { o[k++] = addr; });
}

// device staging -> pinned host address buffer: coalesced 16-B writes over PCIe, size from the scan
__global__ void __launch_bounds__(256) k_addr_copyout(const uint64_t* __restrict__ exp,
                                                      const uint64_t* __restrict__ epos, uint32_t L,
                                                      uint64_t* __restrict__ host_exp) {
  const uint64_t n = epos[L];
  const uint64_t n2 = n / 2;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n2; i += stride)
    reinterpret_cast<ulonglong2*>(host_exp)[i] = reinterpret_cast<const ulonglong2*>(exp)[i];
  if ((n & 1) && blockIdx.x == 0 && threadIdx.x == 0) host_exp[n - 1] = exp[n - 1];
}

__global__ void __launch_bounds__(256) k_lane_caps(uint32_t L, const LaneDesc* __restrict__ lanes, uint32_t elem,
                                                   uint32_t* __restrict__ cap) {
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t < L) cap[t] = lanes[t].nbytes / elem;
}

}  // namespace

void launch_lane_bases(uint32_t L, const LaneDesc* lanes, uint32_t elem, uint32_t* tmp, uint64_t* base,
                       cudaStream_t s) {
  k_lane_caps<<<(L + 255) / 256, 256, 0, s>>>(L, lanes, elem, tmp);
  k_addr_scan<<<1, 1024, 0, s>>>(tmp, L, base, base + L);
}

void launch_addr_stage1(const Chunk& c, const Access& a, const uint64_t* meta, LaneDesc* lanes, uint32_t* tileK,
                        uint32_t elem, uint32_t T, uint32_t pmax, int patterns, const uint64_t* user_addr,
                        const uint64_t* user_base, const uint32_t* user_count, AddrDesc* desc_host,
                        uint32_t* ecount, uint64_t* epos, uint64_t* exp_dev, uint64_t* exp_host,
                        uint64_t* total_host, cudaStream_t s) {
  const AddrSrc src{user_addr, user_base, user_count};
  const uint32_t g = (c.L + 255) / 256;
  k_addr_detect<<<g, 256, 0, s>>>(c, a, meta, lanes, tileK, elem, T, pmax, patterns, src, desc_host, ecount);
  k_addr_scan<<<1, 1024, 0, s>>>(ecount, c.L, epos, total_host);
  k_addr_emit<<<g, 256, 0, s>>>(c, a, meta, lanes, elem, src, ecount, epos, exp_dev);
  k_addr_copyout<<<device_sms(), 256, 0, s>>>(exp_dev, epos, c.L, exp_host);
}

}  // namespace bk
