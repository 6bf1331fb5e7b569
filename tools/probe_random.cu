// Probe (not product code): random-update throughput of HBM on this B200 — the roofline of
// k_kmer's (and k_wc's global) table updates. A table of 2^28 x 16-B entries (4 GiB, far beyond
// the 126 MB L2); each update = read the 8-B key of a random entry, then a fire-and-forget 8-B
// atomic add to its count (k_kmer's hit path). Also: reads only, atomics only.
// nvcc -O3 -gencode arch=compute_100a,code=sm_100a tools/probe_random.cu -o build/probe_random
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint64_t mix64(uint64_t x) {
  x ^= x >> 30; x *= 0xbf58476d1ce4e5b9ULL;
  x ^= x >> 27; x *= 0x94d049bb133111ebULL;
  x ^= x >> 31;
  return x;
}

struct Entry { unsigned long long key, count; };

template <int kMode>  // 0: load key + atomic add count, 1: load only, 2: atomic add only
__global__ void k_rand(Entry* t, uint64_t mask, int iters, unsigned long long seed, unsigned long long* sink) {
  const uint64_t tid = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  unsigned long long acc = 0;
  for (int i = 0; i < iters; ++i) {
    const uint64_t s = mix64(seed ^ (tid * 0x9E3779B97F4A7C15ull + i)) & mask;
    if (kMode != 2) acc += *reinterpret_cast<volatile unsigned long long*>(&t[s].key);
    if (kMode != 1) atomicAdd(&t[s].count, 1ull + (acc & 1));
  }
  if (acc == 0x123456789ull) *sink = acc;
}

int main() {
  const uint64_t slots = 1ull << 28;
  Entry* t;
  unsigned long long* sink;
  cudaMalloc(&t, slots * sizeof(Entry));
  cudaMalloc(&sink, 8);
  cudaMemset(t, 0, slots * sizeof(Entry));
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const int iters = 64;
  for (int mode = 0; mode < 3; ++mode) {
    for (int bps : {4, 8, 16}) {
      const int grid = 148 * bps, block = 256;
      for (int rep = 0; rep < 3; ++rep) {
        cudaEventRecord(a);
        if (mode == 0) k_rand<0><<<grid, block>>>(t, slots - 1, iters, 1234 + rep, sink);
        if (mode == 1) k_rand<1><<<grid, block>>>(t, slots - 1, iters, 1234 + rep, sink);
        if (mode == 2) k_rand<2><<<grid, block>>>(t, slots - 1, iters, 1234 + rep, sink);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        const double n = (double)grid * block * iters;
        if (rep == 2)
          printf("{\"mode\": \"%s\", \"blocks_per_sm\": %d, \"g_updates_s\": %.2f, \"ms\": %.3f}\n",
                 mode == 0 ? "load+atomic" : mode == 1 ? "load" : "atomic", bps, n / ms / 1e6, ms);
      }
    }
  }
  printf("%s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
