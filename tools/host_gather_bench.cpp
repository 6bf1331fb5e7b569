// Host-only benchmark of the product's CPU assembly (host_gather_chunk) on the C2 grep data set.
// Not product code. g++ -O3 -march=x86-64-v3 -fopenmp -I/usr/local/cuda/include -Ipaper_conf_ipps_mokhtaris14_b200/csrc -Igen
//   tools/host_gather_bench.cpp paper_conf_ipps_mokhtaris14_b200/csrc/host_gather.cpp gen/gen.c -o build/hgb -lpthread
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <string>
#include <vector>

#include "gen.h"
#include "host_gather.h"

int main(int argc, char** argv) {
  using namespace bk;
  const double gib = argc > 1 ? atof(argv[1]) : 16;
  const int threads = argc > 2 ? atoi(argv[2]) : 16;
  const bool pack = argc > 3 && std::string(argv[3]) == "pack";   // host_pack_chunk instead of tiles
  const uint64_t n = gen_grep_count_for_bytes(0xB16C0002, 0, (uint64_t)(gib * (1ull << 30)));
  std::vector<uint64_t> off(n);
  const uint64_t nb = gen_grep_sizes(0xB16C0002, 0, n, off.data());
  std::vector<uint8_t> buf(nb);
  gen_grep_fill(0xB16C0002, 0, n, off.data(), buf.data(), 16);
  HostPool pool(threads);
  HostData d{buf.data(), off.data(), n, nb, 0};
  Access a{};
  a.n_ext = 1; a.ext_off[0] = 16; a.ext_len[0] = 32; a.E = 32;
  const uint64_t per = 2097152;  // records per chunk (64 MiB of keys), 8 records per lane
  std::vector<uint8_t> stage(per * 32 + (per / 8) * 64 + 4096);
  std::vector<uint64_t> f, t;
  for (int rep = 0; rep < 3; ++rep) {
    auto t0 = std::chrono::steady_clock::now();
    for (uint64_t lo = 0; lo < n; lo += per) {
      Chunk c{};
      c.lo = lo; c.hi = std::min(n, lo + per);
      c.base_byte = off[lo]; c.end_byte = c.hi < n ? off[c.hi] : nb;
      c.L = (uint32_t)(((c.hi - lo) / 8 + 31) / 32 * 32); c.ntiles = c.L / 32; c.accessed = (c.hi - lo) * 32;
      if (pack) host_pack_chunk(pool, d, a, c, stage.data(), stage.size());
      else host_gather_chunk(pool, d, a, c, stage.data(), stage.size(), f, t);
    }
    double s = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
    printf("{\"mode\": \"%s\", \"threads\": %d, \"s\": %.4f, \"grec_s\": %.3f}\n", pack ? "pack" : "tiles",
           threads, s, n / s / 1e9);
  }
  return 0;
}
