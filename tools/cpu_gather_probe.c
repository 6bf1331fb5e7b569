// Host-side gather probe (not product code): how fast can this box's cores pack the 32-byte keys
// of the C2 grep records (exact gather, SURVEY §8(d) "cpu" mode) into a contiguous buffer?
// Build: gcc -O3 -march=native -fopenmp tools/cpu_gather_probe.c gen/gen.c -Igen -o build/cpu_gather_probe -lm
#include <omp.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <time.h>

#include "gen.h"

static double now(void) {
  struct timespec t;
  clock_gettime(CLOCK_MONOTONIC, &t);
  return t.tv_sec + t.tv_nsec * 1e-9;
}

int main(int argc, char** argv) {
  double gib = argc > 1 ? atof(argv[1]) : 16;
  uint64_t maxb = (uint64_t)(gib * (1ull << 30));
  uint64_t n = gen_grep_count_for_bytes(0xB16C0002, 0, maxb);
  uint64_t* off = malloc(n * 8);
  uint64_t nb = gen_grep_sizes(0xB16C0002, 0, n, off);
  uint8_t* buf = aligned_alloc(4096, (nb + 4095) / 4096 * 4096);
  double t0 = now();
  gen_grep_fill(0xB16C0002, 0, n, off, buf, omp_get_max_threads());
  printf("{\"gen_s\": %.2f, \"records\": %llu, \"bytes\": %llu}\n", now() - t0, (unsigned long long)n, (unsigned long long)nb);
  uint8_t* dst = aligned_alloc(4096, n * 32);
  memset(dst, 0, n * 32);
  int maxt = omp_get_max_threads();
  for (int th = 1; th <= maxt; th *= 2) {
    for (int rep = 0; rep < 2; ++rep) {
      double a = now();
#pragma omp parallel for num_threads(th) schedule(static, 65536)
      for (uint64_t r = 0; r < n; ++r) memcpy(dst + r * 32, buf + off[r] + 16, 32);
      double dt = now() - a;
      if (rep) printf("{\"threads\": %d, \"grec_s\": %.3f, \"key_gbs\": %.2f, \"logical_gbs\": %.2f}\n", th, n / dt / 1e9,
                      n * 32 / dt / 1e9, nb / dt / 1e9);
    }
  }
  // streaming read bandwidth of the whole data set (all threads)
  double a = now();
  uint64_t acc = 0;
#pragma omp parallel for reduction(^ : acc) schedule(static, 1 << 16)
  for (uint64_t i = 0; i < nb / 8; ++i) acc ^= ((uint64_t*)buf)[i];
  double dt = now() - a;
  printf("{\"host_read_gbs_all_threads\": %.2f, \"x\": %llu}\n", nb / dt / 1e9, (unsigned long long)(acc & 1));
  return 0;
}
