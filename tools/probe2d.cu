// Probe (not product code): can the copy engine gather a fixed-stride field with cudaMemcpy2DAsync
// faster than SM zero-copy loads? Reports field GB/s and records/s for width/pitch combinations.
// nvcc -O3 -gencode arch=compute_100a,code=sm_100a tools/probe2d.cu -o build/probe2d
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdlib>
#include <cstring>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("CUDA %s line %d\n", cudaGetErrorString(e_), __LINE__); exit(1);} } while (0)

int main() {
  const size_t bytes = 4ull << 30;
  void* h = nullptr;
  CK(cudaHostAlloc(&h, bytes, cudaHostAllocPortable));
  memset(h, 1, bytes);
  void* d = nullptr;
  CK(cudaMalloc(&d, 1ull << 30));
  cudaStream_t s; CK(cudaStreamCreate(&s));
  cudaEvent_t a, b; CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b));
  const size_t widths[] = {16, 32, 64, 96};
  const size_t pitches[] = {64, 128, 256};
  for (size_t pitch : pitches)
    for (size_t w : widths) {
      if (w >= pitch) continue;
      const size_t rows = bytes / pitch;
      const size_t rows_per = (1ull << 30) / w;   // device buffer holds packed fields
      size_t done = 0;
      float ms = 0;
      for (int rep = 0; rep < 2; ++rep) {
        CK(cudaEventRecord(a, s));
        done = 0;
        while (done < rows) {
          const size_t r = rows - done < rows_per ? rows - done : rows_per;
          const size_t rr = r > 65535 * 16 ? 65535 * 16 : r;
          CK(cudaMemcpy2DAsync(d, w, (char*)h + done * pitch, pitch, w, rr, cudaMemcpyHostToDevice, s));
          done += rr;
        }
        CK(cudaEventRecord(b, s));
        CK(cudaEventSynchronize(b));
        CK(cudaEventElapsedTime(&ms, a, b));
      }
      printf("{\"pitch\": %zu, \"width\": %zu, \"field_gbs\": %.2f, \"logical_gbs\": %.2f, \"grec_s\": %.3f}\n", pitch, w,
             rows * w / ms / 1e6, bytes / ms / 1e6, rows / ms / 1e6);
    }
  return 0;
}
