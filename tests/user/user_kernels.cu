// Test-only user kernels for bk_run_user (tests/test_gpu_user.py): a caller's own stage-4 kernel
// written against the public staged layout of include/bk.h — no libbk internals. Built by the
// Makefile into tests/user/libbkuser.so; never part of the product.
#include <cuda_runtime.h>
#include <stdint.h>

#include "bk.h"

namespace {

__device__ __forceinline__ uint64_t mix64(uint64_t x) {
  x ^= x >> 30; x *= 0xbf58476d1ce4e5b9ULL;
  x ^= x >> 27; x *= 0x94d049bb133111ebULL;
  x ^= x >> 31;
  return x;
}

__device__ __forceinline__ uint32_t staged_byte(const uint8_t* tile, uint32_t col, uint64_t b) {
  return tile[((b >> 4) * 32 + col) * 16 + (b & 15)];
}

// Order-independent checksum: sum over staged records r of mix64(r) * (1 + sum of r's staged bytes)
__global__ void k_user_sum(bk_chunk_view v, uint32_t E, unsigned long long* acc) {
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= v.lanes) return;
  const bk_lane d = v.lane_desc[t];
  const uint8_t* tile = v.stage + v.tile_base[t >> 5];
  unsigned long long local = 0;
  uint64_t pos = 0;
  for (uint32_t j = 0; j < d.nrec; ++j) {
    const uint64_t r = d.first + j;
    uint64_t len = E;
    if (v.offsets) {
      const uint64_t i = r - v.first_record;
      len = (i + 1 < v.n_records ? v.offsets[i + 1] : v.end_offset) - v.offsets[i];
    }
    uint64_t s = 0;
    for (uint64_t b = 0; b < len; ++b) s += staged_byte(tile, t & 31, pos + b);
    pos += len;
    local += mix64(r) * (s + 1);
  }
  if (local) atomicAdd(acc, local);
}

}  // namespace

struct UserSum {
  unsigned long long* acc;   // device accumulator
  uint32_t E;                // accessed bytes per record (ignored for whole variable-length records)
  int32_t fail_at;           // return non-zero at this chunk index (-1: never)
  uint64_t calls;            // callbacks seen (host)
};

extern "C" int user_sum_chunk(const bk_chunk_view* v, void* stream, void* user) {
  UserSum* u = static_cast<UserSum*>(user);
  if (v->struct_size != sizeof(bk_chunk_view)) return 2;
  ++u->calls;
  if (u->fail_at >= 0 && v->chunk_index == (uint64_t)u->fail_at) return 1;
  k_user_sum<<<(v->lanes + 255) / 256, 256, 0, static_cast<cudaStream_t>(stream)>>>(*v, u->E, u->acc);
  return cudaGetLastError() == cudaSuccess ? 0 : 3;
}
