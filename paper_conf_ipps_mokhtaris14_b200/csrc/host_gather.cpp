// host_gather.cpp — CPU assembly of one chunk into the warp-tile layout (see host_gather.h).
// The lane rule and the tile layout are the ones k_addrgen / k_gather_* implement on the GPU
// (DESIGN.md §1, §2 A4); tests/test_gpu_parity.py checks the staged bytes of every gather mode
// against the layout definition.
#include "host_gather.h"

#include <immintrin.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>

namespace bk {

HostPool::HostPool(int threads) {
  if (threads < 1) threads = 1;
  for (int i = 0; i + 1 < threads; ++i) workers_.emplace_back([this, i] { loop(i); });
}

HostPool::~HostPool() {
  {
    std::lock_guard<std::mutex> g(m_);
    stop_ = true;
  }
  cv_.notify_all();
  for (auto& t : workers_) t.join();
}

void HostPool::loop(int tid) {
  uint64_t seen = 0;
  for (;;) {
    std::function<void(int)> job;
    {
      std::unique_lock<std::mutex> l(m_);
      cv_.wait(l, [&] { return stop_ || gen_ != seen; });
      if (stop_) return;
      seen = gen_;
      job = job_;
    }
    job(tid);
    {
      std::lock_guard<std::mutex> g(m_);
      if (--pending_ == 0) done_.notify_all();
    }
  }
}

void HostPool::run(const std::function<void(int)>& f) {
  {
    std::lock_guard<std::mutex> g(m_);
    job_ = f;
    pending_ = (int)workers_.size();
    ++gen_;
  }
  cv_.notify_all();
  f((int)workers_.size());
  std::unique_lock<std::mutex> l(m_);
  done_.wait(l, [&] { return pending_ == 0; });
}

namespace {

inline uint64_t rstart(const HostData& d, uint64_t r) {
  if (!d.off) return r * d.rec_size;
  return r < d.n ? d.off[r] : d.nbytes;
}

// A(lo, r) of the access spec (k_addrgen's acc_bytes)
inline uint64_t acc(const HostData& d, const Access& a, const Chunk& c, uint64_t r) {
  if (!a.whole) return (r - c.lo) * a.E;
  if (!d.off) return (r - c.lo) * d.rec_size;
  return (r == c.hi ? c.end_byte : d.off[r]) - c.base_byte;
}

// first(t) = min{ r in [lo,hi] : A(lo,r) >= floor(t*A/L) } (k_addrgen's lane_first)
inline uint64_t lane_first(const HostData& d, const Access& a, const Chunk& c, uint64_t t) {
  if (t >= c.L) return c.hi;
  const uint64_t target = t * c.accessed / c.L;
  if (a.whole && d.off) {
    uint64_t lo = c.lo, hi = c.hi;
    while (lo < hi) {
      const uint64_t mid = lo + (hi - lo) / 2;
      if (acc(d, a, c, mid) >= target) hi = mid; else lo = mid + 1;
    }
    return lo;
  }
  const uint64_t per = a.whole ? d.rec_size : a.E;
  if (per == 0) return c.lo;
  const uint64_t k = (target + per - 1) / per;
  return std::min(c.lo + k, c.hi);
}

}  // namespace

uint64_t host_staged_size(const HostData& d, const Access& a, const Chunk& c) {
  uint64_t size = 0;
  uint64_t prev = lane_first(d, a, c, 0);
  for (uint32_t w = 0; w < c.ntiles; ++w) {
    uint64_t K = 0;
    for (uint32_t i = 0; i < 32; ++i) {
      const uint64_t nx = lane_first(d, a, c, (uint64_t)w * 32 + i + 1);
      K = std::max<uint64_t>(K, (acc(d, a, c, nx) - acc(d, a, c, prev) + 15) / 16);
      prev = nx;
    }
    size += 512 * K;
  }
  return size;
}

uint64_t host_gather_chunk(HostPool& pool, const HostData& d, const Access& a, const Chunk& c, uint8_t* stage,
                           uint64_t cap, std::vector<uint64_t>& first, std::vector<uint64_t>& tbase) {
  const uint32_t L = c.L, T = c.ntiles;
  first.resize((size_t)L + 1);
  tbase.resize((size_t)T + 1);
  const int P = pool.size();
  // 1. lane bounds and per-tile K_w (parallel over tiles)
  pool.run([&](int tid) {
    const uint64_t per = (T + P - 1) / P;
    for (uint64_t w = tid * per; w < std::min<uint64_t>(T, (tid + 1) * per); ++w) {
      uint64_t K = 0, prev = lane_first(d, a, c, (uint32_t)(w * 32));
      first[w * 32] = prev;
      for (uint32_t i = 0; i < 32; ++i) {
        const uint64_t t = w * 32 + i;
        const uint64_t nx = lane_first(d, a, c, t + 1);
        first[t + 1] = nx;
        const uint64_t b = acc(d, a, c, nx) - acc(d, a, c, prev);
        K = std::max<uint64_t>(K, (b + 15) / 16);
        prev = nx;
      }
      tbase[w] = K;
    }
  });
  // 2. exclusive scan of 512 * K_w
  uint64_t size = 0;
  for (uint32_t w = 0; w < T; ++w) {
    const uint64_t K = tbase[w];
    tbase[w] = size;
    size += 512 * K;
  }
  tbase[T] = size;
  if (size > cap) return UINT64_MAX;
  // 3. fill: each tile is assembled in a thread-local buffer (lane-outer: every lane's records are
  // read in address order, scattered 16-B stores stay in L1), then streamed to the pinned staging
  // slot with non-temporal 16-B stores (no read-for-ownership; the CPU never reads it again).
  const bool fast = !a.whole && a.n_ext == 1 && (a.E % 16) == 0 && a.E > 0;
  const uint32_t EW = a.E / 16, eo = a.n_ext ? a.ext_off[0] : 0;
  std::atomic<uint32_t> next{0};
  pool.run([&](int) {
    std::vector<__m128i> tl;
    for (;;) {
      const uint32_t w0 = next.fetch_add(16);
      if (w0 >= T) break;
      for (uint32_t w = w0; w < std::min(T, w0 + 16); ++w) {
        const uint64_t K = (tbase[w + 1] - tbase[w]) / 512;
        if (tl.size() < K * 32) tl.resize(K * 32);
        uint8_t* tile = reinterpret_cast<uint8_t*>(tl.data());
        memset(tile, 0, K * 512);
        if (fast) {
          // the tile's lanes are consecutive record ranges: walk them in address order with a
          // software prefetch kPf records ahead across lane boundaries (lanes are only ~8 records)
          constexpr uint64_t kPf = 16;
          const uint64_t r0 = first[(uint64_t)w * 32], r1 = first[(uint64_t)w * 32 + 32];
          auto rsrc = [&](uint64_t r) { return d.base + (d.off ? d.off[r] : r * d.rec_size) + eo; };
          for (uint64_t r = r0; r < std::min(r1, r0 + kPf); ++r) __builtin_prefetch(rsrc(r));
          int i = 0;
          uint64_t lane_end = first[(uint64_t)w * 32 + 1], k = 0;
          for (uint64_t r = r0; r < r1; ++r) {
            while (r >= lane_end) {  // next non-empty lane
              ++i;
              k = 0;
              lane_end = first[(uint64_t)w * 32 + i + 1];
            }
            if (r + kPf < r1) __builtin_prefetch(rsrc(r + kPf));
            const uint8_t* srcp = rsrc(r);
            for (uint32_t m = 0; m < EW; ++m, ++k) memcpy(tile + (k * 32 + i) * 16, srcp + 16 * m, 16);
          }
        }
        for (int i = 0; i < 32 && !fast; ++i) {
          const uint64_t t = (uint64_t)w * 32 + i;
          const uint64_t f = first[t], nr = first[t + 1] - f;
          if (a.whole) {
            const uint64_t nb = acc(d, a, c, first[t + 1]) - acc(d, a, c, f);
            const uint8_t* src = d.base + rstart(d, f);
            for (uint64_t b = 0, k = 0; b < nb; b += 16, ++k)
              memcpy(tile + (k * 32 + i) * 16, src + b, std::min<uint64_t>(16, nb - b));
          } else {
            uint64_t b = 0;
            for (uint64_t j = 0; j < nr; ++j) {
              const uint64_t rs = rstart(d, f + j);
              for (uint32_t e = 0; e < a.n_ext; ++e)
                for (uint32_t x = 0; x < a.ext_len[e]; ++x, ++b)
                  tile[((b / 16) * 32 + i) * 16 + b % 16] = d.base[rs + a.ext_off[e] + x];
            }
          }
        }
        __m128i* dst = reinterpret_cast<__m128i*>(stage + tbase[w]);
        for (uint64_t q = 0; q < K * 32; ++q) _mm_stream_si128(dst + q, tl[q]);
      }
    }
    _mm_sfence();
  });
  return size;
}

// Address mode (BK_GATHER_ADDR): the paper's CPU assembly loop, h_pBuf[i] = *(data + addrBuf[i])
// (Fig. 3), per lane from its pattern (base + periodic strides) or its explicit address
// list, in the lane's access order, written in the warp-tile layout. Reads are merged into runs of
// contiguous elements (with a pattern the CPU reads each lane's data sequentially, §IV.B).
uint64_t host_assemble_addr(HostPool& pool, const HostData& d, uint32_t L, uint32_t elem, const AddrDesc* desc,
                            const uint64_t* exp, uint64_t n_exp, uint8_t* stage, uint64_t cap,
                            std::vector<uint64_t>& epos, std::vector<uint64_t>& tbase) {
  const uint32_t T = L / 32;
  epos.resize((size_t)L + 1);
  tbase.resize((size_t)T + 1);
  for (uint32_t t = 0; t < L; ++t)
    if (desc[t].count == 0xffffffffu) return UINT64_MAX - 1;   // a generator count above its lane's capacity
  uint64_t e = 0, size = 0;
  for (uint32_t w = 0; w < T; ++w) {
    uint64_t K = 0;
    for (uint32_t i = 0; i < 32; ++i) {
      const AddrDesc& dd = desc[w * 32 + i];
      epos[w * 32 + i] = e;
      if (dd.p <= 0) e += dd.count;
      K = std::max<uint64_t>(K, ((uint64_t)dd.count * elem + 15) / 16);
    }
    tbase[w] = size;
    size += 512 * K;
  }
  tbase[T] = size;
  epos[L] = e;
  if (e != n_exp) return UINT64_MAX - 1;   // descriptors and explicit list disagree
  if (size > cap) return UINT64_MAX;
  std::atomic<uint32_t> next{0};
  std::atomic<bool> bad{false};
  pool.run([&](int) {
    for (;;) {
      const uint32_t w0 = next.fetch_add(8);
      if (w0 >= T) break;
      for (uint32_t w = w0; w < std::min(T, w0 + 8); ++w) {
        uint8_t* tile = stage + tbase[w];
        const uint64_t K = (tbase[w + 1] - tbase[w]) / 512;
        for (int i = 0; i < 32; ++i) {
          const uint32_t t = w * 32 + i;
          const AddrDesc& dd = desc[t];
          uint64_t b = 0;   // byte position in the lane's stream
          auto put = [&](const uint8_t* src, uint64_t len) {
            while (len) {
              const uint64_t k = b >> 4, o = b & 15;
              uint8_t* dst = tile + (k * 32 + i) * 16;
              if (o == 0 && len >= 16) {   // whole 16-B words: constant-size copies
                memcpy(dst, src, 16);
                b += 16;
                src += 16;
                len -= 16;
                continue;
              }
              const uint64_t m = std::min<uint64_t>(16 - o, len);
              memcpy(dst + o, src, m);
              b += m;
              src += m;
              len -= m;
            }
          };
          uint64_t run0 = 0, runl = 0;   // current run of contiguous elements
          auto elem_at = [&](uint64_t a) {
            if (a > d.nbytes || elem > d.nbytes - a) { bad = true; return; }
            if (runl && a == run0 + runl) { runl += elem; return; }
            if (runl) put(d.base + run0, runl);
            run0 = a;
            runl = elem;
          };
          if (dd.p == 1 && dd.stride[0] == (int64_t)elem && dd.count) {   // one contiguous run
            const uint64_t len = (uint64_t)dd.count * elem;
            if (dd.base > d.nbytes || len > d.nbytes - dd.base) bad = true;
            else put(d.base + dd.base, len);
          } else if (dd.p > 0) {
            uint64_t a = dd.base;
            for (uint32_t k = 0; k < dd.count; ++k) {
              elem_at(a);
              a += (uint64_t)dd.stride[k % (uint32_t)dd.p];
            }
          } else {
            const uint64_t* x = exp + epos[t];
            for (uint32_t k = 0; k < dd.count; ++k) elem_at(x[k]);
          }
          if (runl) put(d.base + run0, runl);
          // zero the tail of the last word and the lane's holes up to the tile's longest lane
          if (b & 15) memset(tile + ((b >> 4) * 32 + i) * 16 + (b & 15), 0, 16 - (b & 15));
          for (uint64_t k = (b + 15) >> 4; k < K; ++k) memset(tile + (k * 32 + i) * 16, 0, 16);
        }
      }
    }
  });
  return bad ? UINT64_MAX - 1 : size;
}

bool host_packable(const Access& a) { return !a.whole && a.n_ext == 1 && a.E > 0 && (a.E % 16) == 0; }

// One packer thread: grabs of kGrab records from a shared counter, each record's E accessed bytes
// copied in record order. Prefetch: near (into L1) PF records ahead — with END both ends of the
// field (a 32-B key crosses a 64-B line for 3 of 8 record alignments) — and far (into L2) PF2
// records ahead. Distances and the 16-B word count are template constants: the same distances read
// from variables cost 15-24% of the packing rate in the bench (gpurun_out/r02bis3_*).
namespace {
using PackSink = std::function<void(uint64_t, uint64_t)>;
using PackFn = void (*)(const HostData&, uint32_t, uint64_t, uint32_t, const Chunk&, uint8_t*, uint64_t, uint64_t, bool,
                        const PackSink*, std::atomic<uint64_t>&);

// copies one record's EW 16-B words: with W32 (EW even, 32-B aligned destination) as 32-B AVX2
// loads / stores, half the memory instructions of the 16-B loop
template <int EWC, bool W32, bool NT>
inline void copy_field(const uint8_t* sp, uint8_t* op, uint32_t EW) {
  if (W32) {
    const __m256i* s = reinterpret_cast<const __m256i*>(sp);
    __m256i* o = reinterpret_cast<__m256i*>(op);
    for (uint32_t m = 0; m < EW / 2; ++m) {
      if (NT) _mm256_stream_si256(o + m, _mm256_loadu_si256(s + m));
      else _mm256_storeu_si256(o + m, _mm256_loadu_si256(s + m));
    }
  } else {
    const __m128i* s = reinterpret_cast<const __m128i*>(sp);
    __m128i* o = reinterpret_cast<__m128i*>(op);
    for (uint32_t m = 0; m < EW; ++m) {
      if (NT) _mm_stream_si128(o + m, _mm_loadu_si128(s + m));
      else _mm_storeu_si128(o + m, _mm_loadu_si128(s + m));
    }
  }
}

template <int PF, int PF2, bool END, int EWC, bool W32>
void pack_worker(const HostData& d, uint32_t eo, uint64_t E, uint32_t ew, const Chunk& c, uint8_t* dst, uint64_t n,
                 uint64_t kGrab, bool nt, const PackSink* sink, std::atomic<uint64_t>& next) {
  const uint32_t EW = EWC ? (uint32_t)EWC : ew;
  auto src = [&](uint64_t r) { return d.base + (d.off ? d.off[r] : r * d.rec_size) + eo; };
  auto pf = [&](uint64_t r) {
    const uint8_t* p = src(r);
    __builtin_prefetch(p);
    if (END) __builtin_prefetch(p + E - 1);
  };
  for (;;) {
    const uint64_t j0 = next.fetch_add(kGrab);
    if (j0 >= n) break;
    const uint64_t j1 = std::min(n, j0 + kGrab);
    for (uint64_t j = j0; j < std::min<uint64_t>(j1, j0 + PF); ++j) pf(c.lo + j);
    if (PF2)
      for (uint64_t j = j0; j < std::min<uint64_t>(j1, j0 + PF2); ++j) _mm_prefetch((const char*)src(c.lo + j), _MM_HINT_T1);
    if (nt) {
      for (uint64_t j = j0; j < j1; ++j) {
        if (j + PF < j1) pf(c.lo + j + PF);
        if (PF2 && j + PF2 < j1) _mm_prefetch((const char*)src(c.lo + j + PF2), _MM_HINT_T1);
        copy_field<EWC, W32, true>(src(c.lo + j), dst + j * E, EW);
      }
      if (sink) _mm_sfence();
    } else {
      for (uint64_t j = j0; j < j1; ++j) {
        if (j + PF < j1) pf(c.lo + j + PF);
        if (PF2 && j + PF2 < j1) _mm_prefetch((const char*)src(c.lo + j + PF2), _MM_HINT_T1);
        copy_field<EWC, W32, false>(src(c.lo + j), dst + j * E, EW);
      }
    }
    if (sink) (*sink)(j0 * E, (j1 - j0) * E);
  }
  _mm_sfence();
}

template <int PF, int PF2, bool END, bool W32 = false>
PackFn pack_for_ew(uint32_t ew) {
  switch (ew) {
    case 1: return pack_worker<PF, PF2, END, 1, false>;
    case 2: return pack_worker<PF, PF2, END, 2, W32>;
    case 6: return pack_worker<PF, PF2, END, 6, W32>;
    default: return pack_worker<PF, PF2, END, 0, false>;
  }
}

// prefetch configurations {near, far, both ends}; BK_PACK_CFG selects one (sweep knob). In the bench
// (HYBRID, zero-copy gathers running; profiles/r02_packer.md): grep 16/0/- 205.7 GB/s, 8/64/ends
// 208.7, 16/64/ends 210.0, 16/0/ends 199.8, 32/128/ends 205.0, 8/0/ends 201.5; sparse group-by
// 16/0/- 108.9, 8/64/ends 115.3, 16/0/ends 111.5. Default: 8/64/ends.
PackFn pack_fn(uint32_t ew, bool dst32) {
  const char* e = getenv("BK_PACK_CFG");   // read per chunk (one call), so a process can switch
  int cfg = e ? atoi(e) : 2;
  if (cfg >= 7 && !dst32) cfg = 2;   // 32-B stores need a 32-B aligned destination
  switch (cfg) {
    case 1: return pack_for_ew<16, 0, false>(ew);   // round 1
    case 3: return pack_for_ew<16, 64, true>(ew);
    case 4: return pack_for_ew<16, 0, true>(ew);
    case 5: return pack_for_ew<32, 128, true>(ew);
    case 6: return pack_for_ew<8, 0, true>(ew);
    // 32-B AVX2 copies (round 2, interleaved on one box, gpurun_out/r02u): grep 200.1-201.5 GB/s vs
    // 208.2-211.1 with the default 16-B loop; sparse group-by (16-B fields, no 32-B path) unchanged
    case 7: return pack_for_ew<8, 64, true, true>(ew);
    case 8: return pack_for_ew<16, 64, true, true>(ew);
    default: return pack_for_ew<8, 64, true>(ew);
  }
}
}  // namespace

uint64_t host_pack_chunk(HostPool& pool, const HostData& d, const Access& a, const Chunk& c, uint8_t* dst,
                         uint64_t cap, uint64_t grab, bool nt, const std::function<void(uint64_t, uint64_t)>* sink) {
  const uint64_t E = a.E, n = c.hi - c.lo, size = n * E;
  if (size > cap) return UINT64_MAX;
  const uint32_t eo = a.ext_off[0], EW = (uint32_t)(E / 16);
  // sweep on the 16-core host (profiles/r01_hybrid_sweep.md): grabs of 4k-16k records read in order
  const uint64_t kGrab = grab ? grab : 16384;
  const PackFn fn = pack_fn(EW, ((uintptr_t)dst & 31) == 0);
  std::atomic<uint64_t> next{0};
  pool.run([&](int) { fn(d, eo, E, EW, c, dst, n, kGrab, nt, sink, next); });
  return size;
}

// The runs of bucket b sit at chunk_base[c] + sum_{b' < b} counts[c][b'] in the chunk-major array;
// in the bucket-major order they follow each other in chunk order from bucket_start[b]. Every run
// is one memcpy; threads take runs in blocks from a shared counter (runs average n / (C * B) records).
int partition_materialize(const uint8_t* runs, const uint64_t* counts, uint64_t n_chunks, uint32_t n_buckets,
                          const uint64_t* bucket_start, uint8_t* dst, uint32_t threads) {
  constexpr uint64_t R = 16;  // bytes per {key, value} record
  struct Run { uint64_t src, dst, n; };
  std::vector<uint64_t> bstart(n_buckets), bnext(n_buckets);
  if (bucket_start) {
    for (uint32_t b = 0; b < n_buckets; ++b) bstart[b] = bucket_start[b];
  } else {
    std::vector<uint64_t> tot(n_buckets, 0);
    for (uint64_t c = 0; c < n_chunks; ++c)
      for (uint32_t b = 0; b < n_buckets; ++b) tot[b] += counts[c * n_buckets + b];
    uint64_t acc = 0;
    for (uint32_t b = 0; b < n_buckets; ++b) { bstart[b] = acc; acc += tot[b]; }
  }
  bnext = bstart;
  std::vector<Run> work;
  work.reserve((size_t)std::min<uint64_t>(n_chunks * n_buckets, 1u << 24));
  uint64_t src = 0;
  for (uint64_t c = 0; c < n_chunks; ++c)
    for (uint32_t b = 0; b < n_buckets; ++b) {
      const uint64_t m = counts[c * n_buckets + b];
      if (m) work.push_back({src, bnext[b], m});
      src += m;
      bnext[b] += m;
    }
  unsigned T = threads ? threads : std::max(1u, std::thread::hardware_concurrency());
  T = (unsigned)std::min<uint64_t>(T, std::max<size_t>(work.size() / 16, 1));
  std::atomic<size_t> next{0};
  auto body = [&]() {
    for (;;) {
      const size_t i0 = next.fetch_add(16);
      if (i0 >= work.size()) return;
      for (size_t i = i0; i < std::min(work.size(), i0 + 16); ++i)
        memcpy(dst + work[i].dst * R, runs + work[i].src * R, work[i].n * R);
    }
  };
  std::vector<std::thread> pool;
  for (unsigned t = 1; t < T; ++t) pool.emplace_back(body);
  body();
  for (auto& th : pool) th.join();
  return 0;
}

}  // namespace bk
