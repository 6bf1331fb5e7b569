// kernels_baseline.cu — the paper's GPU double-buffering baseline (variant iv, PAPER.md P:994-996;
// host loop P:329-339; kernel form P:313-318): raw chunks of whole records are copied into one of
// two device buffers and the unchanged kernel runs on them, each thread over a contiguous record
// range (myParticleStartIndex .. EndIndex). No address generation, no assembly, no interleaving.
// Used only as the measured comparison point (BK_FLAG_BASELINE_DBUF); same results as the
// BigKernel path.
#include "bk_internal.cuh"

namespace bk {
namespace {

constexpr unsigned kFull = 0xffffffffu;

struct RawChunk {
  const uint8_t* raw;      // byte base_byte of the data set
  const uint64_t* meta;    // offsets slice (NULL: fixed records)
  uint64_t lo, hi, base_byte, end_byte, rec_size;
};

__device__ __forceinline__ uint64_t rstart(const RawChunk& c, uint64_t r) {
  if (!c.meta) return r * c.rec_size - c.base_byte;
  return (r == c.hi ? c.end_byte : c.meta[r - c.lo]) - c.base_byte;
}

// thread t of T owns records [lo + t*n/T, lo + (t+1)*n/T)
__device__ __forceinline__ void my_range(const RawChunk& c, uint64_t& a, uint64_t& b) {
  const uint64_t T = (uint64_t)gridDim.x * blockDim.x, t = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  const uint64_t n = c.hi - c.lo;
  a = c.lo + n * t / T;
  b = c.lo + n * (t + 1) / T;
}

__device__ bool raw_match(const RawChunk& c, uint64_t r, const uint8_t* pat, uint32_t plen) {
  const uint8_t* k = c.raw + rstart(c, r) + 16;
  uint32_t kl = 0;
  while (kl < 32 && k[kl]) ++kl;
  if (plen == 0) return true;
  for (uint32_t p = 0; p + plen <= kl; ++p) {
    uint32_t q = 0;
    while (q < plen && k[p + q] == pat[q]) ++q;
    if (q == plen) return true;
  }
  return false;
}

struct Pat { uint8_t b[32]; uint32_t len; };

__global__ void __launch_bounds__(256) k_dbuf_grep_count(RawChunk c, Pat pat, uint32_t* blkcnt) {
  __shared__ uint32_t ws[8];
  uint64_t a, b;
  my_range(c, a, b);
  uint32_t n = 0;
  for (uint64_t r = a; r < b; ++r) n += raw_match(c, r, pat.b, pat.len);
  n = __reduce_add_sync(kFull, n);
  if ((threadIdx.x & 31) == 0) ws[threadIdx.x >> 5] = n;
  __syncthreads();
  if (threadIdx.x == 0) {
    uint32_t s = 0;
    for (int i = 0; i < 8; ++i) s += ws[i];
    blkcnt[blockIdx.x] = s;
  }
}

__global__ void __launch_bounds__(256) k_dbuf_grep_write(RawChunk c, Pat pat, const unsigned long long* blkbase,
                                                         uint64_t first_index, uint64_t* out, uint64_t cap) {
  __shared__ uint32_t ws[8];
  uint64_t a, b;
  my_range(c, a, b);
  uint32_t n = 0;
  for (uint64_t r = a; r < b; ++r) n += raw_match(c, r, pat.b, pat.len);
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  uint32_t x = n;
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(kFull, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) ws[w] = x;
  __syncthreads();
  uint32_t before = 0;
  for (int i = 0; i < w; ++i) before += ws[i];
  unsigned long long pos = blkbase[blockIdx.x] + before + x - n;
  if (n)
    for (uint64_t r = a; r < b; ++r)
      if (raw_match(c, r, pat.b, pat.len)) {
        if (pos < cap) out[pos] = first_index + r;
        ++pos;
      }
}

// running += sum(blkcnt); blkbase = exclusive scan + old running (one block)
__global__ void __launch_bounds__(1024) k_dbuf_scan(const uint32_t* blkcnt, uint32_t nblk, unsigned long long* running,
                                                    unsigned long long* blkbase) {
  __shared__ unsigned long long carry;
  if (threadIdx.x == 0) {
    unsigned long long s = *running;
    for (uint32_t i = 0; i < nblk; ++i) {
      blkbase[i] = s;
      s += blkcnt[i];
    }
    carry = s;
    *running = carry;
  }
}

__global__ void __launch_bounds__(256) k_dbuf_groupby(RawChunk c, uint32_t G, unsigned long long* gcount,
                                                      unsigned long long* gqty, double* gamount, int* err) {
  extern __shared__ unsigned char smem_raw[];
  double* s_amt = reinterpret_cast<double*>(smem_raw);
  unsigned int* s_cnt = reinterpret_cast<unsigned int*>(s_amt + G);
  unsigned int* s_qty = s_cnt + G;
  for (uint32_t g = threadIdx.x; g < G; g += blockDim.x) { s_amt[g] = 0.0; s_cnt[g] = 0; s_qty[g] = 0; }
  __syncthreads();
  uint64_t a, b;
  my_range(c, a, b);
  for (uint64_t r = a; r < b; ++r) {
    const uint8_t* p = c.raw + rstart(c, r);
    const uint32_t key = *reinterpret_cast<const uint32_t*>(p);
    if (key >= G) { atomicOr(err, kErrKeyRange); continue; }
    atomicAdd(&s_cnt[key], 1u);
    atomicAdd(&s_qty[key], *reinterpret_cast<const uint32_t*>(p + 4));
    atomicAdd(&s_amt[key], *reinterpret_cast<const double*>(p + 8));
  }
  __syncthreads();
  for (uint32_t g = threadIdx.x; g < G; g += blockDim.x)
    if (s_cnt[g]) {
      atomicAdd(&gcount[g], (unsigned long long)s_cnt[g]);
      atomicAdd(&gqty[g], (unsigned long long)s_qty[g]);
      atomicAdd(&gamount[g], s_amt[g]);
    }
}

// K-means step on raw 64-B+ records (16 fp32 at +0), thread per contiguous record range, the
// distance / argmin / accumulation rules of k_kmeans (A13) on the original AoS layout.
__global__ void __launch_bounds__(256) k_dbuf_kmeans(RawChunk c, const float* __restrict__ mu, uint32_t K,
                                                     uint64_t first_index, unsigned long long* gcount, double* gsum,
                                                     unsigned long long* gchk) {
  extern __shared__ unsigned char smem_raw[];
  double* s_sum = reinterpret_cast<double*>(smem_raw);
  float* s_mu = reinterpret_cast<float*>(s_sum + (size_t)K * 16);
  unsigned int* s_cnt = reinterpret_cast<unsigned int*>(s_mu + (size_t)K * 16);
  for (uint32_t i = threadIdx.x; i < K * 16; i += blockDim.x) { s_sum[i] = 0.0; s_mu[i] = mu[i]; }
  for (uint32_t i = threadIdx.x; i < K; i += blockDim.x) s_cnt[i] = 0;
  __syncthreads();
  uint64_t a, b;
  my_range(c, a, b);
  unsigned long long chk = 0;
  for (uint64_t r = a; r < b; ++r) {
    const float4* p = reinterpret_cast<const float4*>(c.raw + rstart(c, r));
    float x[16];
    for (int w = 0; w < 4; ++w) {
      const float4 v = p[w];
      x[4 * w] = v.x; x[4 * w + 1] = v.y; x[4 * w + 2] = v.z; x[4 * w + 3] = v.w;
    }
    uint32_t best = 0;
    float bestd = 0.0f;
    for (uint32_t k = 0; k < K; ++k) {
      float acc = 0.0f;
      for (int q = 0; q < 16; ++q) {
        const float df = __fsub_rn(x[q], s_mu[k * 16 + q]);
        acc = __fmaf_rn(df, df, acc);
      }
      if (k == 0 || acc < bestd) { bestd = acc; best = k; }
    }
    atomicAdd(&s_cnt[best], 1u);
    for (int q = 0; q < 16; ++q) atomicAdd(&s_sum[best * 16 + q], (double)x[q]);
    chk += mix64(((first_index + r) << 8) ^ (uint64_t)best);
  }
  for (int o = 16; o; o >>= 1) chk += __shfl_xor_sync(kFull, chk, o);
  __syncthreads();
  for (uint32_t i = threadIdx.x; i < K * 16; i += blockDim.x)
    if (s_sum[i] != 0.0) atomicAdd(&gsum[i], s_sum[i]);
  for (uint32_t i = threadIdx.x; i < K; i += blockDim.x)
    if (s_cnt[i]) atomicAdd(&gcount[i], (unsigned long long)s_cnt[i]);
  if ((threadIdx.x & 31) == 0) atomicAdd(gchk, chk);
}

}  // namespace

uint32_t dbuf_blocks() { return (uint32_t)device_sms() * 4; }

void launch_dbuf_kmeans(const uint8_t* raw, uint64_t lo, uint64_t hi, uint64_t base_byte, uint64_t rec_size,
                        const float* mu, uint32_t K, uint64_t first_index, unsigned long long* count, double* sum,
                        unsigned long long* chk, cudaStream_t s) {
  RawChunk c{raw, nullptr, lo, hi, base_byte, hi * rec_size, rec_size};
  const size_t smem = (size_t)K * 16 * 12 + (size_t)K * 4;
  k_dbuf_kmeans<<<dbuf_blocks(), 256, smem, s>>>(c, mu, K, first_index, count, sum, chk);
}

void launch_dbuf_grep(const uint8_t* raw, const uint64_t* meta, uint64_t lo, uint64_t hi, uint64_t base_byte,
                      uint64_t end_byte, uint64_t rec_size, const GrepParams& p, uint32_t* blkcnt,
                      unsigned long long* running, unsigned long long* blkbase, uint64_t* out, cudaStream_t s) {
  RawChunk c{raw, meta, lo, hi, base_byte, end_byte, rec_size};
  Pat pat{};
  for (uint32_t i = 0; i < p.plen; ++i) pat.b[i] = p.pat[i];
  pat.len = p.plen;
  const uint32_t nb = dbuf_blocks();
  k_dbuf_grep_count<<<nb, 256, 0, s>>>(c, pat, blkcnt);
  k_dbuf_scan<<<1, 32, 0, s>>>(blkcnt, nb, running, blkbase);
  k_dbuf_grep_write<<<nb, 256, 0, s>>>(c, pat, blkbase, p.first_index, out, p.cap);
}

void launch_dbuf_groupby(const uint8_t* raw, uint64_t lo, uint64_t hi, uint64_t base_byte, uint64_t rec_size,
                         uint32_t G, unsigned long long* count, unsigned long long* qty, double* amount, int* err,
                         cudaStream_t s) {
  RawChunk c{raw, nullptr, lo, hi, base_byte, hi * rec_size, rec_size};
  k_dbuf_groupby<<<dbuf_blocks(), 256, (size_t)G * 16, s>>>(c, G, count, qty, amount, err);
}

cudaError_t configure_baseline_kernels() {
  const cudaError_t e = cudaFuncSetAttribute(k_dbuf_groupby, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  if (e != cudaSuccess) return e;
  return cudaFuncSetAttribute(k_dbuf_kmeans, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
}

}  // namespace bk
