// Phase-0 box probe: host-link and zero-copy bandwidths.
// Not product code. Build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a tools/probe.cu -o build/probe
#include <cuda_runtime.h>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <cstdint>
#include <vector>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { \
  fprintf(stderr, "CUDA %s at %s:%d\n", cudaGetErrorString(e_), __FILE__, __LINE__); exit(1);} } while (0)

// Coalesced zero-copy read of a contiguous host range: each thread 16-B loads, UNROLL in flight.
template <int UNROLL>
__global__ void zc_seq(const uint4* __restrict__ src, size_t nwords, uint4* sink) {
  size_t tid = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
  size_t stride = (size_t)gridDim.x * blockDim.x;
  uint4 acc = make_uint4(0, 0, 0, 0);
  for (size_t base = tid; base < nwords; base += stride * UNROLL) {
    uint4 v[UNROLL];
#pragma unroll
    for (int u = 0; u < UNROLL; ++u) {
      size_t i = base + (size_t)u * stride;
      v[u] = i < nwords ? __ldcs(src + i) : make_uint4(0, 0, 0, 0);
    }
#pragma unroll
    for (int u = 0; u < UNROLL; ++u) { acc.x ^= v[u].x; acc.y ^= v[u].y; acc.z ^= v[u].z; acc.w ^= v[u].w; }
  }
  if ((acc.x ^ acc.y ^ acc.z ^ acc.w) == 0x12345678u) sink[0] = acc;
}

// Sparse zero-copy read: one `bytes`-long field (16-B aligned) per `rec` bytes, one record per thread.
template <int W>
__global__ void zc_sparse(const uint8_t* __restrict__ src, size_t nrec, size_t rec, uint4* sink) {
  size_t tid = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
  size_t stride = (size_t)gridDim.x * blockDim.x;
  uint4 acc = make_uint4(0, 0, 0, 0);
  for (size_t r = tid; r < nrec; r += stride) {
    const uint4* p = reinterpret_cast<const uint4*>(src + r * rec);
#pragma unroll
    for (int w = 0; w < W; ++w) { uint4 v = __ldcs(p + w); acc.x ^= v.x; acc.y ^= v.y; }
  }
  if ((acc.x ^ acc.y) == 0x12345678u) sink[0] = acc;
}

static double now() {
  return std::chrono::duration<double>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

int main(int argc, char** argv) {
  size_t gib = argc > 1 ? atoll(argv[1]) : 8;
  size_t bytes = gib << 30;
  CK(cudaSetDevice(0));
  cudaDeviceProp prop; CK(cudaGetDeviceProperties(&prop, 0));
  printf("{\"device\": \"%s\", \"sms\": %d, \"pci\": \"%04x:%02x:%02x\"}\n", prop.name, prop.multiProcessorCount,
         prop.pciDomainID, prop.pciBusID, prop.pciDeviceID);
  void* h = nullptr;
  double t0 = now();
  h = aligned_alloc(1 << 21, bytes);
  memset(h, 1, bytes);
  double t1 = now();
  CK(cudaHostRegister(h, bytes, cudaHostRegisterMapped | cudaHostRegisterPortable));
  double t2 = now();
  printf("{\"host_touch_gib_s\": %.2f, \"host_register_s_per_gib\": %.4f}\n", gib / (t1 - t0), (t2 - t1) / gib);
  void* d = nullptr; CK(cudaMalloc(&d, bytes > (8ull << 30) ? (8ull << 30) : bytes));
  size_t dbytes = bytes > (8ull << 30) ? (8ull << 30) : bytes;
  cudaStream_t s1, s2; CK(cudaStreamCreate(&s1)); CK(cudaStreamCreate(&s2));
  cudaEvent_t a, b; CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b));
  // H2D at several chunk sizes
  for (size_t chunk : {1ull << 20, 4ull << 20, 16ull << 20, 64ull << 20, 256ull << 20}) {
    for (int rep = 0; rep < 2; ++rep) {
      CK(cudaEventRecord(a, s1));
      for (size_t off = 0; off < dbytes; off += chunk)
        CK(cudaMemcpyAsync((char*)d + off, (char*)h + off, chunk, cudaMemcpyHostToDevice, s1));
      CK(cudaEventRecord(b, s1)); CK(cudaEventSynchronize(b));
      float ms; CK(cudaEventElapsedTime(&ms, a, b));
      if (rep) printf("{\"h2d_chunk_mib\": %zu, \"gbs\": %.2f}\n", chunk >> 20, dbytes / ms / 1e6);
    }
  }
  // D2H
  {
    CK(cudaEventRecord(a, s1));
    for (size_t off = 0; off < dbytes; off += 64 << 20)
      CK(cudaMemcpyAsync((char*)h + off, (char*)d + off, 64 << 20, cudaMemcpyDeviceToHost, s1));
    CK(cudaEventRecord(b, s1)); CK(cudaEventSynchronize(b));
    float ms; CK(cudaEventElapsedTime(&ms, a, b));
    printf("{\"d2h_gbs\": %.2f}\n", dbytes / ms / 1e6);
  }
  // Bidirectional
  {
    size_t half = dbytes / 2;
    double w0 = now();
    for (size_t off = 0; off < half; off += 64 << 20) {
      CK(cudaMemcpyAsync((char*)d + off, (char*)h + off, 64 << 20, cudaMemcpyHostToDevice, s1));
      CK(cudaMemcpyAsync((char*)h + half + off, (char*)d + half + off, 64 << 20, cudaMemcpyDeviceToHost, s2));
    }
    CK(cudaDeviceSynchronize());
    double w1 = now();
    printf("{\"bidir_each_dir_gbs\": %.2f}\n", half / (w1 - w0) / 1e9);
  }
  uint8_t* hd = nullptr; CK(cudaHostGetDevicePointer((void**)&hd, h, 0));
  uint4* sink; CK(cudaMalloc(&sink, 64));
  int grids[] = {148, 296, 592, 1184, 2368};
  for (int g : grids) {
    for (int blk : {256, 512}) {
      size_t nw = dbytes / 16;
      for (int rep = 0; rep < 2; ++rep) {
        CK(cudaEventRecord(a, s1));
        zc_seq<4><<<g, blk, 0, s1>>>((const uint4*)hd, nw, sink);
        CK(cudaEventRecord(b, s1)); CK(cudaEventSynchronize(b));
        float ms; CK(cudaEventElapsedTime(&ms, a, b));
        if (rep) printf("{\"zc_seq_grid\": %d, \"block\": %d, \"gbs\": %.2f}\n", g, blk, dbytes / ms / 1e6);
      }
    }
  }
  for (size_t rec : {64ull, 128ull, 256ull}) {
    size_t nrec = dbytes / rec;
    for (int w : {1, 2, 4}) {
      if ((size_t)w * 16 > rec) continue;
      float ms = 0;
      for (int rep = 0; rep < 2; ++rep) {
        CK(cudaEventRecord(a, s1));
        if (w == 1) zc_sparse<1><<<1184, 512, 0, s1>>>(hd, nrec, rec, sink);
        if (w == 2) zc_sparse<2><<<1184, 512, 0, s1>>>(hd, nrec, rec, sink);
        if (w == 4) zc_sparse<4><<<1184, 512, 0, s1>>>(hd, nrec, rec, sink);
        CK(cudaEventRecord(b, s1)); CK(cudaEventSynchronize(b));
        CK(cudaEventElapsedTime(&ms, a, b));
      }
      printf("{\"zc_sparse_rec\": %zu, \"field_bytes\": %d, \"field_gbs\": %.2f, \"logical_gbs\": %.2f, \"rec_per_s_g\": %.3f}\n",
             rec, w * 16, nrec * w * 16 / ms / 1e6, dbytes / ms / 1e6, nrec / ms / 1e6);
    }
  }
  CK(cudaGetLastError());
  return 0;
}
