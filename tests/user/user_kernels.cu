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

// ---- bk_run_user_addr: a caller-written stage 1 (address generator) and its stage-4 consumer ----
namespace {

// Fixed records: lane t emits, for its records in REVERSE order, every `step`-th `elem`-byte element
// of the field [ext_off, ext_off + ext_len) — an access order the pattern recogniser sees as a
// negative-stride walk when step == 1 within a record, and as explicit addresses across records.
__global__ void k_gen_fixed(bk_addr_view v, uint32_t rec_size, uint32_t ext_off, uint32_t ext_len, uint32_t step) {
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= v.lanes) return;
  const bk_lane d = v.lane_desc[t];
  const uint32_t m = (ext_len / v.elem_bytes + step - 1) / step;   // elements per record
  uint64_t* out = v.addr + v.addr_base[t];
  uint32_t k = 0;
  for (uint32_t j = 0; j < d.nrec; ++j) {
    const uint64_t r = d.first + d.nrec - 1 - j;
    for (uint32_t e = 0; e < m; ++e) out[k++] = r * rec_size + ext_off + (uint64_t)e * step * v.elem_bytes;
  }
  v.addr_count[t] = k;
}

// Variable records (grep layout): per record, the 8-byte id at +8 AFTER the first 8 key bytes at +16
__global__ void k_gen_var(bk_addr_view v) {
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= v.lanes) return;
  const bk_lane d = v.lane_desc[t];
  uint64_t* out = v.addr + v.addr_base[t];
  uint32_t k = 0;
  for (uint32_t j = 0; j < d.nrec; ++j) {
    const uint64_t rs = v.offsets[d.first + j - v.first_record];
    out[k++] = rs + 16;
    out[k++] = rs + 8;
  }
  v.addr_count[t] = k;
}

__global__ void k_gen_bad(bk_addr_view v, uint64_t bad_addr, uint32_t over) {
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= v.lanes) return;
  const uint32_t cap = (uint32_t)(v.lane_desc[t].nbytes / v.elem_bytes);
  if (t == 0 && over) { v.addr_count[t] = cap + 1; return; }
  if (t == 0 && cap) { v.addr[v.addr_base[t]] = bad_addr; v.addr_count[t] = 1; return; }
  v.addr_count[t] = 0;
}

// Consumer: element k of lane t is 8 bytes (or 4); checksum sum mix64(tag(t, k)) * (value + 1) where
// tag is the (record, element) the generator assigned to position k.
__global__ void k_use_fixed(bk_chunk_view v, uint32_t ext_len, uint32_t step, uint32_t elem, unsigned long long* acc) {
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= v.lanes) return;
  const bk_lane d = v.lane_desc[t];
  const uint8_t* tile = v.stage + v.tile_base[t >> 5];
  const uint32_t m = (ext_len / elem + step - 1) / step;
  const uint32_t n = d.nbytes / elem;
  unsigned long long local = 0;
  for (uint32_t k = 0; k < n; ++k) {
    uint64_t val = 0;
    for (uint32_t q = 0; q < elem; ++q) val |= (uint64_t)staged_byte(tile, t & 31, (uint64_t)k * elem + q) << (8 * q);
    const uint64_t r = d.first + d.nrec - 1 - k / m, e = (uint64_t)(k % m) * step;
    local += mix64((r << 8) ^ e) * (val + 1);
  }
  if (local) atomicAdd(acc, local);
}

__global__ void k_use_var(bk_chunk_view v, unsigned long long* acc) {
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= v.lanes) return;
  const bk_lane d = v.lane_desc[t];
  const uint8_t* tile = v.stage + v.tile_base[t >> 5];
  unsigned long long local = 0;
  for (uint32_t j = 0; j < d.nbytes / 16; ++j) {
    uint64_t key = 0, id = 0;
    for (uint32_t q = 0; q < 8; ++q) {
      key |= (uint64_t)staged_byte(tile, t & 31, 16ull * j + q) << (8 * q);
      id |= (uint64_t)staged_byte(tile, t & 31, 16ull * j + 8 + q) << (8 * q);
    }
    local += mix64(d.first + j) * ((key ^ id) + 1);
  }
  if (local) atomicAdd(acc, local);
}

}  // namespace

struct UserGen {
  uint32_t rec_size, ext_off, ext_len, step;   // k_gen_fixed; rec_size == 0: k_gen_var
  int32_t mode;                               // 0 normal, 1 out-of-range address, 2 count over capacity
  uint32_t _pad;
  uint64_t bad_addr;
};
struct UserUse {
  unsigned long long* acc;
  uint32_t ext_len, step, elem, variable;
};

extern "C" int user_gen(const bk_addr_view* v, void* stream, void* user) {
  const UserGen* g = static_cast<const UserGen*>(user);
  if (v->struct_size != sizeof(bk_addr_view)) return 2;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  const uint32_t grid = (v->lanes + 255) / 256;
  if (g->mode) k_gen_bad<<<grid, 256, 0, s>>>(*v, g->bad_addr, g->mode == 2);
  else if (g->rec_size) k_gen_fixed<<<grid, 256, 0, s>>>(*v, g->rec_size, g->ext_off, g->ext_len, g->step);
  else k_gen_var<<<grid, 256, 0, s>>>(*v);
  return cudaGetLastError() == cudaSuccess ? 0 : 3;
}

extern "C" int user_use(const bk_chunk_view* v, void* stream, void* user) {
  const UserUse* u = static_cast<const UserUse*>(user);
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  const uint32_t grid = (v->lanes + 255) / 256;
  if (u->variable) k_use_var<<<grid, 256, 0, s>>>(*v, u->acc);
  else k_use_fixed<<<grid, 256, 0, s>>>(*v, u->ext_len, u->step, u->elem, u->acc);
  return cudaGetLastError() == cudaSuccess ? 0 : 3;
}
