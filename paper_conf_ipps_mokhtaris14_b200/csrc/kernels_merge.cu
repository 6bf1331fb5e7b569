// kernels_merge.cu — the multi-GPU merge of per-GPU count tables (word count and
// k-mer tables are all-gathered over NCCL into one device buffer, then merged by key here).
//
// The paper is single-GPU; records are independent segments, so sharding them over GPUs
// changes nothing but where each partial table lives, and the merged table is the per-key sum.
// One thread per gathered row inserts it into an open-addressing table of row indices:
//   owner[s] = smallest gathered row index whose key hashes to probe chain position s (claimed by
//              atomicCAS, lowered by atomicMin among equal keys: the FIRST row in (segment, row)
//              order, i.e. the lowest rank's payload, whatever the thread schedule),
//   cnt[s]   = sum of the counts of every row with that key (atomicAdd).
// Keys are compared word by word against the owner's row, which is immutable input, so no
// publication protocol is needed. A second pass writes one merged row per occupied slot.
#include "bk_internal.cuh"

namespace bk {
namespace {

constexpr unsigned long long kEmpty = ~0ull;
constexpr int kMaxRow = 16;

__device__ __forceinline__ uint64_t key_hash(const uint64_t* r, uint32_t key_u64) {
  uint64_t h = 0x243F6A8885A308D3ull;
  for (uint32_t i = 0; i < key_u64; ++i) h = mix64(h ^ (r[i] + 0x9E3779B97F4A7C15ull * (i + 1)));
  return h;
}

__device__ __forceinline__ bool key_eq(const uint64_t* a, const uint64_t* b, uint32_t key_u64) {
  for (uint32_t i = 0; i < key_u64; ++i)
    if (a[i] != b[i]) return false;
  return true;
}

struct SegRows {
  uint64_t n[64];
};

// grid.y = segment; grid-stride over that segment's valid rows
__global__ void __launch_bounds__(256) k_merge_insert(const uint64_t* __restrict__ rows, uint64_t seg_stride,
                                                      SegRows seg, uint32_t row_u64, uint32_t key_u64,
                                                      uint32_t count_col, unsigned long long* owner,
                                                      unsigned long long* cnt, uint64_t mask, int* err) {
  const uint32_t sg = blockIdx.y;
  const uint64_t nrow = seg.n[sg];
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < nrow; i += (uint64_t)gridDim.x * blockDim.x) {
    const unsigned long long g = sg * seg_stride + i;
    const uint64_t* r = rows + g * row_u64;
    const unsigned long long c = r[count_col];
    uint64_t s = key_hash(r, key_u64) & mask;
    bool done = false;
    for (uint64_t probe = 0; probe <= mask; ++probe, s = (s + 1) & mask) {
      unsigned long long o = atomicCAS(&owner[s], kEmpty, g);
      if (o == kEmpty || key_eq(rows + o * row_u64, r, key_u64)) {
        if (o != kEmpty) atomicMin(&owner[s], g);
        atomicAdd(&cnt[s], c);
        done = true;
        break;
      }
    }
    if (!done) atomicOr(err, kErrTableFull);
  }
}

__global__ void __launch_bounds__(256) k_merge_emit(const uint64_t* __restrict__ rows, uint32_t row_u64,
                                                    uint32_t count_col, const unsigned long long* __restrict__ owner,
                                                    const unsigned long long* __restrict__ cnt, uint64_t slots,
                                                    uint64_t* __restrict__ out, uint64_t cap,
                                                    unsigned long long* n_out) {
  for (uint64_t s = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; s < slots; s += (uint64_t)gridDim.x * blockDim.x) {
    const unsigned long long o = owner[s];
    if (o == kEmpty) continue;
    const unsigned long long p = atomicAdd(n_out, 1ull);
    if (p >= cap) continue;
    const uint64_t* r = rows + o * row_u64;
    uint64_t* w = out + p * row_u64;
    for (uint32_t j = 0; j < row_u64; ++j) w[j] = j == count_col ? cnt[s] : r[j];
  }
}

}  // namespace

cudaError_t launch_merge_counts(const uint64_t* rows, uint32_t n_seg, uint64_t seg_stride, const uint64_t* seg_rows,
                                uint32_t row_u64, uint32_t key_u64, uint32_t count_col, unsigned long long* owner,
                                unsigned long long* cnt, uint64_t slots, uint64_t* out, uint64_t cap,
                                unsigned long long* n_out, int* err, cudaStream_t s) {
  if (n_seg > 64 || row_u64 > kMaxRow) return cudaErrorInvalidValue;
  SegRows sr{};
  uint64_t most = 0;
  for (uint32_t i = 0; i < n_seg; ++i) {
    sr.n[i] = seg_rows[i];
    most = most > seg_rows[i] ? most : seg_rows[i];
  }
  cudaError_t e;
  if ((e = cudaMemsetAsync(owner, 0xff, slots * 8, s)) != cudaSuccess) return e;
  if ((e = cudaMemsetAsync(cnt, 0, slots * 8, s)) != cudaSuccess) return e;
  if ((e = cudaMemsetAsync(n_out, 0, 8, s)) != cudaSuccess) return e;
  const int sms = device_sms();
  if (most && n_seg) {
    const uint64_t want = (most + 255) / 256;
    const uint32_t gx = (uint32_t)(want < (uint64_t)sms * 4 ? want : (uint64_t)sms * 4);
    k_merge_insert<<<dim3(gx, n_seg), 256, 0, s>>>(rows, seg_stride, sr, row_u64, key_u64, count_col, owner, cnt,
                                                   slots - 1, err);
  }
  k_merge_emit<<<sms * 4, 256, 0, s>>>(rows, row_u64, count_col, owner, cnt, slots, out, cap, n_out);
  return cudaGetLastError();
}

}  // namespace bk
