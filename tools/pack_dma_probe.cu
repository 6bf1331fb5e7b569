// Probe (not product code): host packing of the C2 grep keys + H2D DMA, the CPU leg of the HYBRID
// pipeline in isolation. Compares one DMA per packed 64-MiB chunk (current) with DMAs issued by
// the packing threads per grab while the bytes are still cache-hot, NT vs regular stores.
// nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -Xcompiler -march=x86-64-v3,-fopenmp
//   -Ipaper_conf_ipps_mokhtaris14_b200/csrc -Igen tools/pack_dma_probe.cu
//   paper_conf_ipps_mokhtaris14_b200/csrc/host_gather.cpp gen/gen.c -o build/pdp -lpthread -lgomp
#include <cuda_runtime.h>

#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <mutex>
#include <string>
#include <vector>

#include "gen.h"
#include "host_gather.h"

#define CK(x)                                                                  \
  do {                                                                         \
    cudaError_t e_ = (x);                                                      \
    if (e_ != cudaSuccess) {                                                   \
      fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e_)); \
      exit(1);                                                                 \
    }                                                                          \
  } while (0)

int main(int argc, char** argv) {
  using namespace bk;
  const double gib = argc > 1 ? atof(argv[1]) : 16;
  const int threads = argc > 2 ? atoi(argv[2]) : 16;
  const uint64_t n = gen_grep_count_for_bytes(0xB16C0002, 0, (uint64_t)(gib * (1ull << 30)));
  std::vector<uint64_t> off(n);
  const uint64_t nb = gen_grep_sizes(0xB16C0002, 0, n, off.data());
  uint8_t* buf = (uint8_t*)aligned_alloc(4096, (nb + 4095) / 4096 * 4096);
  gen_grep_fill(0xB16C0002, 0, n, off.data(), buf, 16);
  HostPool pool(threads);
  HostData d{buf, off.data(), n, nb, 0};
  Access a{};
  a.n_ext = 1; a.ext_off[0] = 16; a.ext_len[0] = 32; a.E = 32;
  const uint64_t per = 2097152;  // records per chunk (64 MiB of keys)
  const uint64_t cap = per * 32;
  const int NH = 3;
  uint8_t* hs[NH];
  cudaEvent_t done[NH];
  for (int i = 0; i < NH; ++i) {
    CK(cudaHostAlloc((void**)&hs[i], cap, cudaHostAllocPortable));
    CK(cudaEventCreateWithFlags(&done[i], cudaEventDisableTiming));
  }
  uint8_t* dev;
  CK(cudaMalloc(&dev, 2 * cap));
  cudaStream_t st;
  CK(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking));
  struct Mode { const char* name; bool nt; bool per_grab; uint64_t grab; };
  const Mode modes[] = {{"nt_one_dma", true, false, 16384},   {"nt_grab_dma_16k", true, true, 16384},
                        {"reg_one_dma", false, false, 16384}, {"reg_grab_dma_16k", false, true, 16384},
                        {"reg_grab_dma_64k", false, true, 65536}, {"reg_grab_dma_4k", false, true, 4096}};
  std::mutex mu;
  for (const Mode& m : modes) {
    for (int rep = 0; rep < 2; ++rep) {
      bool used[NH] = {false, false, false};
      CK(cudaDeviceSynchronize());
      auto t0 = std::chrono::steady_clock::now();
      double pack_s = 0;
      uint64_t k = 0;
      for (uint64_t lo = 0; lo < n; lo += per, ++k) {
        const int h = (int)(k % NH);
        if (used[h]) CK(cudaEventSynchronize(done[h]));
        Chunk c{};
        c.lo = lo; c.hi = std::min(n, lo + per);
        uint8_t* dst = dev + (k & 1) * cap;
        std::function<void(uint64_t, uint64_t)> sink = [&](uint64_t o, uint64_t b) {
          std::lock_guard<std::mutex> g(mu);
          CK(cudaMemcpyAsync(dst + o, hs[h] + o, b, cudaMemcpyHostToDevice, st));
        };
        auto p0 = std::chrono::steady_clock::now();
        const uint64_t size = host_pack_chunk(pool, d, a, c, hs[h], cap, m.grab, m.nt, m.per_grab ? &sink : nullptr);
        pack_s += std::chrono::duration<double>(std::chrono::steady_clock::now() - p0).count();
        if (!m.per_grab) CK(cudaMemcpyAsync(dst, hs[h], size, cudaMemcpyHostToDevice, st));
        CK(cudaEventRecord(done[h], st));
        used[h] = true;
      }
      CK(cudaStreamSynchronize(st));
      const double s = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
      if (rep)
        printf("{\"mode\": \"%s\", \"threads\": %d, \"s\": %.4f, \"grec_s\": %.3f, \"pack_grec_s\": %.3f, \"gbs_logical\": %.1f}\n",
               m.name, threads, s, n / s / 1e9, n / pack_s / 1e9, nb / s / 1e9);
      fflush(stdout);
    }
  }
  return 0;
}
