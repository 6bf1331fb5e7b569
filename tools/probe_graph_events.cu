// Not product code. Do timing events recorded inside a captured CUDA graph carry timestamps?
// nvcc -O2 -gencode arch=compute_100a,code=sm_100a tools/probe_graph_events.cu -o build/probe_graph_events
#include <cstdio>
#include <cuda_runtime.h>
__global__ void spin(long long ns) {
  long long t0 = clock64();
  while (clock64() - t0 < ns * 2) {}
}
int main() {
  cudaStream_t s, s2;
  cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking);
  cudaEvent_t a, b, c, fork, join;
  cudaEventCreate(&a); cudaEventCreate(&b); cudaEventCreate(&c);
  cudaEventCreateWithFlags(&fork, cudaEventDisableTiming); cudaEventCreateWithFlags(&join, cudaEventDisableTiming);
  cudaGraph_t g; cudaGraphExec_t ge;
  cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal);
  cudaEventRecord(a, s);
  spin<<<1, 1, 0, s>>>(100000);        // ~100 us
  cudaEventRecord(b, s);
  cudaEventRecord(fork, s);
  cudaStreamWaitEvent(s2, fork, 0);
  spin<<<1, 1, 0, s2>>>(200000);       // ~200 us on a side stream
  cudaEventRecord(c, s2);
  cudaEventRecord(join, s2);
  cudaStreamWaitEvent(s, join, 0);
  cudaError_t e = cudaStreamEndCapture(s, &g);
  printf("capture: %s\n", cudaGetErrorString(e));
  e = cudaGraphInstantiate(&ge, g, 0);
  printf("instantiate: %s\n", cudaGetErrorString(e));
  for (int it = 0; it < 3; ++it) {
    e = cudaGraphLaunch(ge, s);
    cudaStreamSynchronize(s);
    float ab = -1, ac = -1;
    cudaError_t r1 = cudaEventElapsedTime(&ab, a, b);
    cudaError_t r2 = cudaEventElapsedTime(&ac, a, c);
    printf("launch %d: %s  a->b %.3f ms (%s)  a->c %.3f ms (%s)\n", it, cudaGetErrorString(e), ab,
           cudaGetErrorString(r1), ac, cudaGetErrorString(r2));
  }
  return 0;
}
