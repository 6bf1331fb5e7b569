// bk_runtime.cu — host runtime of libbk: context, registration (pin once), chunk planner,
// ring of N staging slots driven by events across copy / assembly / compute streams, and the
// C ABI of include/bk.h.
//
// Paper mapping (Fig. 3, §III, §IV.C):
//   * pinned buffers      -> the data set itself is pinned + mapped ONCE at
//                                        registration; device staging is allocated once at create;
//   * wait_addrReady / signal_dataReady flags -> cudaEvents per slot;
//   * "at minimum two" buffer instances, addr-gen n syncs with compute n-3
//                                     -> a ring of N slots; chunk c reuses slot c % N only after
//                                        the compute of chunk c - N recorded slot_free;
//   * CPU assembly thread per block -> replaced by a GPU gather kernel that reads
//                                        pinned host memory directly (zero-copy) or by a DMA of
//                                        the whole chunk followed by an HBM re-layout kernel.
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <new>
#include <string>
#include <thread>
#include <vector>

#include "../../include/bk.h"
#include "bk_internal.cuh"
#include "host_gather.h"

using namespace bk;

namespace {

thread_local std::string g_last_error;

int fail(int code, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  g_last_error = buf;
  return code;
}

#define BK_CUDA(expr)                                                                        \
  do {                                                                                       \
    cudaError_t e_ = (expr);                                                                 \
    if (e_ != cudaSuccess)                                                                   \
      return fail(BK_E_CUDA, "%s failed: %s (%s:%d)", #expr, cudaGetErrorString(e_), __FILE__, __LINE__); \
  } while (0)

constexpr uint64_t kAlign = 256;
inline uint64_t align_up(uint64_t x, uint64_t a) { return (x + a - 1) / a * a; }

struct Slot {
  uint8_t* raw = nullptr;       // DENSE: the chunk's record bytes as DMA'd
  uint8_t* stage = nullptr;     // interleaved warp tiles
  uint64_t* meta = nullptr;     // offsets slice off[lo .. hi-1]
  LaneDesc* lanes = nullptr;
  uint32_t* tileK = nullptr;
  uint64_t* tile_base = nullptr;
  uint8_t* out = nullptr;       // per-chunk output (partition: the bucket-sorted chunk)
  cudaEvent_t copied = nullptr, ready = nullptr, freed = nullptr;
  bool used = false;
};

// Resident (outside the window) per-kernel device buffers, grown on demand.
struct DevBuf {
  void* p = nullptr;
  size_t cap = 0;
  cudaError_t ensure(size_t bytes) {
    if (bytes <= cap) return cudaSuccess;
    if (p) cudaFree(p);
    p = nullptr;
    cap = 0;
    cudaError_t e = cudaMalloc(&p, bytes);
    if (e == cudaSuccess) cap = bytes;
    return e;
  }
  void release() {
    if (p) cudaFree(p);
    p = nullptr;
    cap = 0;
  }
};

// A run plan: depends only on the registration, the access spec and the config, so it is
// computed once and cached per context (plan_cache) until the next registration.
struct Plan {
  Access a{};
  int mode = BK_GATHER_DENSE;          // resolved gather mode
  int zero_copy = 0;                   // plan budget counts accessed bytes (every mode but DENSE)
  uint64_t budget = 0;                 // plan bytes per chunk
  uint32_t L = 0;
  uint64_t max_acc_rec = 0;            // max accessed bytes of one record
  uint64_t stage_cap = 0, raw_cap = 0, meta_cap = 0, out_cap = 0;
  std::vector<uint64_t> bounds;        // chunk record bounds
  std::string key;                     // plan-cache key (also part of the graph key)
};

// A captured pipeline (CUDA graph) for one (kernel, parameters, plan, output pointers), replayed
// by later bk_run calls with the same key instead of re-issuing ~10 launches/copies per chunk.
struct GraphEntry {
  std::string key;
  cudaGraphExec_t exec = nullptr;
  bk_stats st{};
  int n_launch = 0;
  size_t prof_used = 0;
  std::vector<int> prof_stage;
};

}  // namespace

struct bk_ctx {
  bk_config cfg{};
  cudaStream_t s_copy = nullptr, s_asm = nullptr, s_comp = nullptr;
  std::vector<cudaStream_t> s_slot;  // per-slot compute streams for commutative kernels
  cudaEvent_t ev_begin = nullptr, ev_end = nullptr;
  cudaEvent_t t_begin = nullptr, t_end = nullptr;   // timing events on s_comp (device time of a run)
  std::vector<cudaEvent_t> prof;                   // BK_FLAG_PROFILE: per chunk x stage begin/end
  std::vector<int> prof_stage;                     // stage id of each event pair
  size_t prof_used = 0;
  uint8_t* window = nullptr;    // the whole streaming working set (cfg.window_bytes)
  std::vector<Slot> slots;
  // registration
  const uint8_t* host = nullptr;
  uint64_t nbytes = 0;
  const uint64_t* off = nullptr;
  uint64_t n = 0;
  bool pinned_data = false, pinned_off = false, registered = false;
  const uint8_t* host_dev = nullptr;   // device alias of the mapped data set
  uint64_t max_rec = 0, min_rec = 0;
  // device scratch / resident buffers
  int* d_err = nullptr;
  unsigned long long* d_ctr = nullptr;  // [0] staged sum, [1] wc used, [2] wc n_out, [3] grep running, [4] kmeans chk
  DevBuf b_table, b_out1, b_out2, b_out3, b_blk, b_blk2, b_agg1, b_agg2, b_agg3, b_mu;
  // CPU assembly (BK_GATHER_CPU / HYBRID): thread pool + pinned host staging ring
  HostPool* pool = nullptr;
  std::vector<uint8_t*> hstage;
  std::vector<cudaEvent_t> h_done;
  std::vector<bool> h_used;
  uint64_t hstage_cap = 0;
  uint64_t h_next = 0;
  std::vector<uint64_t> scratch_first, scratch_tiles;
  // partition: D2H stream, per-slot "kernels done" events, resident totals, pinned output cache
  cudaStream_t s_d2h = nullptr;
  std::vector<cudaEvent_t> ev_part;
  DevBuf b_hist, b_colpre, b_totals, b_base;
  std::vector<std::pair<void*, uint64_t>> out_pinned;  // caller output arrays this context pinned
  int n_launch = 0;
  bk_stats st{};
  std::vector<std::pair<std::string, Plan>> plan_cache;
  std::vector<GraphEntry> graphs;
  cudaEvent_t ev_fork = nullptr;
  std::vector<cudaEvent_t> ev_join;
  float* h_mu = nullptr;   // pinned copy of the k-means centroids (graph memcpy source)
  uint64_t test_rng = 0x9E3779B97F4A7C15ull;   // BK_FLAG_TEST_DELAYS
};

namespace {

bool is_pinned(const void* p) {
  cudaPointerAttributes at;
  if (cudaPointerGetAttributes(&at, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return at.type == cudaMemoryTypeHost;
}

uint64_t rec_start(const bk_ctx* c, uint64_t r) {
  if (!c->off) return r * c->cfg.record_size;
  return r < c->n ? c->off[r] : c->nbytes;
}

// plan bytes of records [lo, r): what the budget limits (DESIGN.md §Chunk plan)
uint64_t plan_bytes(const bk_ctx* c, const Plan& p, uint64_t lo, uint64_t r) {
  if (!p.zero_copy || p.a.whole) return rec_start(c, r) - rec_start(c, lo);
  return (r - lo) * p.a.E;
}

int make_chunks(const bk_ctx* c, Plan& p) {
  p.bounds.clear();
  p.bounds.push_back(0);
  uint64_t lo = 0;
  const bool fixed_per = !c->off || (p.zero_copy && !p.a.whole);
  const uint64_t per = !c->off ? (p.zero_copy && !p.a.whole ? p.a.E : c->cfg.record_size) : p.a.E;
  while (lo < c->n) {
    uint64_t hi;
    if (fixed_per) {
      if (per > p.budget) return fail(BK_E_RANGE, "record (%llu B) exceeds chunk budget (%llu B)",
                                      (unsigned long long)per, (unsigned long long)p.budget);
      hi = per ? std::min<uint64_t>(c->n, lo + p.budget / per) : c->n;
    } else {
      const uint64_t limit = c->off[lo] + p.budget;
      if (c->nbytes <= limit) {
        hi = c->n;
      } else {
        // first r > lo with off[r] > limit, then hi = r - 1
        const uint64_t* it = std::upper_bound(c->off + lo + 1, c->off + c->n, limit);
        hi = (uint64_t)(it - c->off) - 1;
      }
      if (hi == lo) return fail(BK_E_RANGE, "record %llu (%llu B) exceeds chunk budget (%llu B)",
                                (unsigned long long)lo, (unsigned long long)(rec_start(c, lo + 1) - rec_start(c, lo)),
                                (unsigned long long)p.budget);
    }
    p.bounds.push_back(hi);
    lo = hi;
  }
  return BK_OK;
}

// Bytes one slot needs for a plan: raw + stage + meta + lanes + tiles (+ alignment).
uint64_t slot_need(const Plan& p) {
  const uint64_t ntiles = p.L / 32;
  return align_up(p.raw_cap, kAlign) + align_up(p.stage_cap, kAlign) + align_up(p.meta_cap * 8, kAlign) +
         align_up((uint64_t)p.L * sizeof(LaneDesc), kAlign) + align_up(ntiles * 4, kAlign) +
         align_up((ntiles + 1) * 8, kAlign) + align_up(p.out_cap, kAlign);
}

void size_plan(const bk_ctx* c, Plan& p, uint64_t budget, uint32_t lane_target) {
  p.budget = budget;
  // largest accessed byte count of any chunk of this plan (dense mode plans by whole records,
  // so with sparse or duplicated extents accessed != planned bytes)
  uint64_t acc = 0, maxrecs = 0;
  for (size_t i = 0; i + 1 < p.bounds.size(); ++i) {
    const uint64_t lo = p.bounds[i], hi = p.bounds[i + 1];
    const uint64_t a = p.a.whole ? rec_start(c, hi) - rec_start(c, lo) : (hi - lo) * p.a.E;
    acc = std::max(acc, a);
    maxrecs = std::max(maxrecs, hi - lo);
  }
  uint32_t L = c->cfg.lanes;
  if (!L) {
    uint64_t l = (acc + lane_target - 1) / lane_target;
    l = (l + 31) / 32 * 32;
    L = (uint32_t)std::max<uint64_t>(32, std::min<uint64_t>(l, 1u << 22));
  }
  p.L = L;
  // staged <= A + L*(max record + 32): DESIGN.md §Stage-1 bound. For whole variable-length records
  // (word count) that worst case is ~2x the payload, so size the slot from the exact staged size of
  // every chunk instead (the k_addrgen lane rule evaluated on the host over the offsets).
  p.stage_cap = align_up(acc + (uint64_t)L * (p.max_acc_rec + 32) + 512, 512);
  if (p.a.whole && c->off && p.bounds.size() > 1) {
    HostData d{c->host, c->off, c->n, c->nbytes, 0};
    Access a = p.a;
    a.rec_size = 0;
    uint64_t mx = 0;
    for (size_t i = 0; i + 1 < p.bounds.size(); ++i) {
      Chunk ch{};
      ch.lo = p.bounds[i];
      ch.hi = p.bounds[i + 1];
      ch.base_byte = rec_start(c, ch.lo);
      ch.end_byte = rec_start(c, ch.hi);
      ch.L = L;
      ch.ntiles = L / 32;
      ch.accessed = ch.end_byte - ch.base_byte;
      mx = std::max(mx, host_staged_size(d, a, ch));
    }
    p.stage_cap = align_up(mx + 512, 512);
  }
  p.raw_cap = p.zero_copy ? 0 : budget + 64;
  p.meta_cap = c->off ? maxrecs + 1 : 0;
}

int plan_run_uncached(bk_ctx* c, const Access& a, uint32_t lane_target, Plan& p, uint32_t out_per_rec,
                      int auto_mode) {
  p.a = a;
  if (c->cfg.lane_bytes) lane_target = c->cfg.lane_bytes;
  int mode = (int)c->cfg.gather_mode;
  // AUTO (counters in profiles/): whole-record access -> DENSE (copy engine at
  // 55.5 GB/s beats zero-copy's 51.4); sparse access -> HYBRID (host assembly packs exactly the
  // accessed bytes; the zero-copy gather is request-rate bound and only adds capacity on top).
  if (mode == BK_GATHER_AUTO) mode = auto_mode != BK_GATHER_AUTO ? auto_mode : a.whole ? BK_GATHER_DENSE : BK_GATHER_HYBRID;
  if (mode != BK_GATHER_ZC && mode != BK_GATHER_DENSE && mode != BK_GATHER_CPU && mode != BK_GATHER_HYBRID)
    return fail(BK_E_INVAL, "bad gather_mode %d", mode);
  p.mode = mode;
  p.zero_copy = mode != BK_GATHER_DENSE;
  p.max_acc_rec = a.whole ? c->max_rec : a.E;
  const uint64_t slot = c->cfg.window_bytes / c->cfg.n_slots;
  // total plan bytes
  const uint64_t total = (p.zero_copy && !a.whole) ? c->n * a.E : c->nbytes;
  uint64_t budget = c->cfg.chunk_bytes;
  bool autob = budget == 0;
  if (autob) {
    // >= ~32 chunks so pipeline fill/drain is a few percent, >= 1 MiB each, and fit a slot
    budget = std::max<uint64_t>(total / 32, 1ull << 20);
    budget = std::min<uint64_t>(budget, slot);
  }
  for (int iter = 0; iter < 64; ++iter) {
    p.budget = budget;
    int rc = make_chunks(c, p);
    if (rc) return rc;
    size_plan(c, p, budget, lane_target);
    uint64_t maxrecs = 0;  // per-chunk output buffer: out_per_rec bytes per record (partition, cid)
    for (size_t i = 0; i + 1 < p.bounds.size(); ++i) maxrecs = std::max<uint64_t>(maxrecs, p.bounds[i + 1] - p.bounds[i]);
    p.out_cap = maxrecs * out_per_rec;
    if (slot_need(p) <= slot) return BK_OK;
    if (!autob) break;
    budget = budget * 3 / 4;
    if (budget < p.max_acc_rec || budget < 16) break;
  }
  return fail(BK_E_NOMEM, "window of %llu B (%u slots) cannot hold a chunk of %llu B (need %llu B per slot)",
              (unsigned long long)c->cfg.window_bytes, c->cfg.n_slots, (unsigned long long)budget,
              (unsigned long long)slot_need(p));
}

int plan_run(bk_ctx* c, const Access& a, uint32_t lane_target, Plan& p, uint32_t out_per_chunk = 0,
             int auto_mode = BK_GATHER_AUTO) {
  char key[256];
  snprintf(key, sizeof key, "%u/%u/%u/%u/%u/%u/%u/%u/%u/%u/%d/%d", a.whole, a.n_ext, a.ext_off[0], a.ext_len[0],
           a.ext_off[1], a.ext_len[1], a.ext_off[2], a.ext_len[2], a.E, lane_target, (int)out_per_chunk, auto_mode);
  std::string k(key);
  for (uint32_t e = 3; e < a.n_ext; ++e) k += "/" + std::to_string(a.ext_off[e]) + ":" + std::to_string(a.ext_len[e]);
  for (auto& kv : c->plan_cache)
    if (kv.first == k) {
      p = kv.second;
      return BK_OK;
    }
  const int rc = plan_run_uncached(c, a, lane_target, p, out_per_chunk, auto_mode);
  p.key = k;
  if (rc == BK_OK) c->plan_cache.emplace_back(k, p);
  return rc;
}

void carve(bk_ctx* c, const Plan& p) {
  const uint64_t slot = c->cfg.window_bytes / c->cfg.n_slots;
  const uint64_t ntiles = p.L / 32;
  for (uint32_t i = 0; i < c->cfg.n_slots; ++i) {
    uint8_t* q = c->window + i * slot;
    Slot& s = c->slots[i];
    s.raw = p.raw_cap ? q : nullptr;
    q += align_up(p.raw_cap, kAlign);
    s.stage = q;
    q += align_up(p.stage_cap, kAlign);
    s.meta = reinterpret_cast<uint64_t*>(q);
    q += align_up(p.meta_cap * 8, kAlign);
    s.lanes = reinterpret_cast<LaneDesc*>(q);
    q += align_up((uint64_t)p.L * sizeof(LaneDesc), kAlign);
    s.tileK = reinterpret_cast<uint32_t*>(q);
    q += align_up(ntiles * 4, kAlign);
    s.tile_base = reinterpret_cast<uint64_t*>(q);
    q += align_up((ntiles + 1) * 8, kAlign);
    s.out = p.out_cap ? q : nullptr;
    s.used = false;
  }
}

Chunk chunk_of(const bk_ctx* c, const Plan& p, size_t i) {
  Chunk ch{};
  ch.lo = p.bounds[i];
  ch.hi = p.bounds[i + 1];
  ch.base_byte = rec_start(c, ch.lo);
  ch.end_byte = rec_start(c, ch.hi);
  ch.L = p.L;
  ch.ntiles = p.L / 32;
  ch.accessed = p.a.whole ? ch.end_byte - ch.base_byte : (ch.hi - ch.lo) * p.a.E;
  return ch;
}

// BK_FLAG_PROFILE: bracket one stage of one chunk with timing events on its stream.
// stage ids of the profiling events: transfer = {H2D, Gather (zero-copy)}, compute = {Compute}
enum { kStH2D = 0, kStAddrgen = 1, kStGather = 2, kStCompute = 3, kStRelayout = 4, kNStages = 5 };
int prof_mark(bk_ctx* c, int stage, cudaStream_t s, bool begin) {
  if (!(c->cfg.flags & BK_FLAG_PROFILE)) return BK_OK;
  if (begin) {
    if (c->prof_used + 2 > c->prof.size()) {
      for (int k = 0; k < 64; ++k) {
        cudaEvent_t e;
        BK_CUDA(cudaEventCreate(&e));
        c->prof.push_back(e);
        if (c->prof.size() % 2 == 0) c->prof_stage.push_back(0);
      }
    }
    c->prof_stage[c->prof_used / 2] = stage;
    BK_CUDA(cudaEventRecord(c->prof[c->prof_used], s));
  } else {
    BK_CUDA(cudaEventRecord(c->prof[c->prof_used + 1], s));
    c->prof_used += 2;
  }
  return BK_OK;
}
#define BK_PROF(stage, stream, begin) do { int r_ = prof_mark(c, stage, stream, begin); if (r_) return r_; } while (0)

// BK_FLAG_TEST_DELAYS: a random spin kernel (0..~100 us) on the stream before every stage, so a
// missing event dependency between stages shows up as wrong results (SURVEY §4 delay injection).
uint64_t test_rand(bk_ctx* c) {
  c->test_rng = c->test_rng * 6364136223846793005ull + 1442695040888963407ull;
  return c->test_rng >> 33;
}
#define BK_DELAY(stream)                                                        \
  do {                                                                          \
    if (c->cfg.flags & BK_FLAG_TEST_DELAYS) launch_spin((long long)(test_rand(c) % 200000), stream); \
  } while (0)

int ensure_host_side(bk_ctx* c, const Plan& p) {
  if (!c->pool) {
    int th = (int)c->cfg.host_threads;
    if (th <= 0) th = (int)std::max(1u, std::thread::hardware_concurrency());
    c->pool = new (std::nothrow) HostPool(th);
    if (!c->pool) return fail(BK_E_NOMEM, "host pool");
  }
  const size_t NH = 3;
  if (c->hstage_cap < p.stage_cap || c->hstage.size() != NH) {
    for (auto* h : c->hstage) cudaFreeHost(h);
    c->hstage.assign(NH, nullptr);
    for (auto& h : c->hstage) BK_CUDA(cudaHostAlloc((void**)&h, p.stage_cap, cudaHostAllocPortable));
    c->hstage_cap = p.stage_cap;
    if (c->h_done.empty()) {
      c->h_done.assign(NH, nullptr);
      for (auto& e : c->h_done) BK_CUDA(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    }
  }
  c->h_used.assign(NH, false);
  c->h_next = 0;
  return BK_OK;
}

// CPU assembly of chunk i (stage 2 on the host pool) + one DMA of the packed tiles (stage 3).
int stage_chunk_cpu(bk_ctx* c, const Plan& p, size_t i, Slot& s) {
  const Chunk ch = chunk_of(c, p, i);
  Access a = p.a;
  a.rec_size = c->off ? 0 : c->cfg.record_size;
  const size_t hs = c->h_next++ % c->hstage.size();
  if (c->h_used[hs]) BK_CUDA(cudaEventSynchronize(c->h_done[hs]));   // its previous DMA finished
  if (c->cfg.flags & BK_FLAG_TEST_DELAYS)   // host-side jitter before the assembly
    std::this_thread::sleep_for(std::chrono::microseconds(test_rand(c) % 200));
  const auto t0 = std::chrono::steady_clock::now();
  HostData d{c->host, c->off, c->n, c->nbytes, c->cfg.record_size};
  const uint64_t size = host_gather_chunk(*c->pool, d, a, ch, c->hstage[hs], p.stage_cap, c->scratch_first,
                                          c->scratch_tiles);
  c->st.ms_cpu_gather += std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  if (size == UINT64_MAX) return fail(BK_E_RANGE, "host-staged chunk exceeds its slot (internal bound violated)");
  if (s.used) BK_CUDA(cudaStreamWaitEvent(c->s_copy, s.freed, 0));
  BK_DELAY(c->s_copy);
    BK_PROF(kStH2D, c->s_copy, true);
  if (c->off && a.whole && ch.hi > ch.lo) {  // record boundaries for whole-record kernels
    BK_CUDA(cudaMemcpyAsync(s.meta, c->off + ch.lo, (ch.hi - ch.lo) * 8, cudaMemcpyHostToDevice, c->s_copy));
    c->st.bytes_meta += (ch.hi - ch.lo) * 8;
  }
  if (size) BK_CUDA(cudaMemcpyAsync(s.stage, c->hstage[hs], size, cudaMemcpyHostToDevice, c->s_copy));
  BK_CUDA(cudaEventRecord(c->h_done[hs], c->s_copy));
  c->h_used[hs] = true;
  BK_PROF(kStH2D, c->s_copy, false);
  BK_PROF(kStAddrgen, c->s_copy, true);
  launch_addrgen(ch, a, s.meta, s.lanes, s.tileK, s.tile_base, p.stage_cap, c->d_err, c->d_ctr + 0, c->s_copy);
  BK_PROF(kStAddrgen, c->s_copy, false);
  c->n_launch += 2;
  c->st.bytes_h2d += size;   // payload + tile padding (A9: padding crosses the link only in this mode)
  c->st.bytes_accessed += ch.accessed;
  c->st.n_chunks_cpu += 1;
  BK_CUDA(cudaEventRecord(s.ready, c->s_copy));
  s.used = true;
  return BK_OK;
}

// Stages 1-3 of chunk i into slot s (on s_copy / s_asm); records s.ready.
int stage_chunk(bk_ctx* c, const Plan& p, size_t i, Slot& s) {
  const Chunk ch = chunk_of(c, p, i);
  Access a = p.a;
  a.rec_size = c->off ? 0 : c->cfg.record_size;
  if (p.zero_copy) {
    // Stage 1 on s_asm (offsets slice by DMA + lane plan) runs ahead, overlapping the previous
    // chunk's zero-copy gather on s_copy; the gather waits only for its own plan.
    if (s.used) BK_CUDA(cudaStreamWaitEvent(c->s_asm, s.freed, 0));
    BK_DELAY(c->s_asm);
    BK_PROF(kStH2D, c->s_asm, true);
    if (c->off && ch.hi > ch.lo) {
      BK_CUDA(cudaMemcpyAsync(s.meta, c->off + ch.lo, (ch.hi - ch.lo) * 8, cudaMemcpyHostToDevice, c->s_asm));
      c->st.bytes_meta += (ch.hi - ch.lo) * 8;
    }
    BK_PROF(kStH2D, c->s_asm, false);
    BK_PROF(kStAddrgen, c->s_asm, true);
    launch_addrgen(ch, a, s.meta, s.lanes, s.tileK, s.tile_base, p.stage_cap, c->d_err, c->d_ctr + 0, c->s_asm);
    BK_PROF(kStAddrgen, c->s_asm, false);
    BK_CUDA(cudaEventRecord(s.copied, c->s_asm));
    BK_CUDA(cudaStreamWaitEvent(c->s_copy, s.copied, 0));
    BK_DELAY(c->s_copy);
    BK_PROF(kStGather, c->s_copy, true);
    Chunk gch = ch;   // readable source: the registered data set
    gch.guard_lo = ch.base_byte;
    gch.guard_hi = c->nbytes - ch.base_byte;
    launch_gather(gch, a, c->host_dev + ch.base_byte, s.meta, s.lanes, s.tile_base, s.stage, p.stage_cap, 1,
                  c->s_copy);
    BK_PROF(kStGather, c->s_copy, false);
    c->n_launch += 3;
    c->st.bytes_h2d += ch.accessed;
  } else {
    if (s.used) BK_CUDA(cudaStreamWaitEvent(c->s_copy, s.freed, 0));
    BK_DELAY(c->s_copy);
    BK_PROF(kStH2D, c->s_copy, true);
    if (c->off && ch.hi > ch.lo) {
      BK_CUDA(cudaMemcpyAsync(s.meta, c->off + ch.lo, (ch.hi - ch.lo) * 8, cudaMemcpyHostToDevice, c->s_copy));
      c->st.bytes_meta += (ch.hi - ch.lo) * 8;
    }
    const uint64_t raw_off = ((uintptr_t)(c->host + ch.base_byte)) & 15;
    const uint64_t bytes = ch.end_byte - ch.base_byte;
    if (bytes) BK_CUDA(cudaMemcpyAsync(s.raw + raw_off, c->host + ch.base_byte, bytes, cudaMemcpyHostToDevice, c->s_copy));
    BK_PROF(kStH2D, c->s_copy, false);
    BK_CUDA(cudaEventRecord(s.copied, c->s_copy));
    BK_CUDA(cudaStreamWaitEvent(c->s_asm, s.copied, 0));
    BK_PROF(kStAddrgen, c->s_asm, true);
    launch_addrgen(ch, a, s.meta, s.lanes, s.tileK, s.tile_base, p.stage_cap, c->d_err, c->d_ctr + 0, c->s_asm);
    BK_PROF(kStAddrgen, c->s_asm, false);
    BK_DELAY(c->s_asm);
    BK_PROF(kStRelayout, c->s_asm, true);
    Chunk gch = ch;   // readable source: the raw slot (256-B aligned, 64 B of slack)
    gch.guard_lo = raw_off;
    gch.guard_hi = p.raw_cap - raw_off;
    launch_gather(gch, a, s.raw + raw_off, s.meta, s.lanes, s.tile_base, s.stage, p.stage_cap, 0, c->s_asm);
    BK_PROF(kStRelayout, c->s_asm, false);
    c->n_launch += 3;
    c->st.bytes_h2d += bytes;
  }
  c->st.bytes_accessed += ch.accessed;
  BK_CUDA(cudaEventRecord(s.ready, p.zero_copy ? c->s_copy : c->s_asm));
  s.used = true;
  return BK_OK;
}

void note_plan(bk_ctx* c, const Plan& p) {
  c->st.gather_mode = (uint32_t)p.mode;
  c->st.chunk_budget = p.budget;
  c->st.lanes = p.L;
}

int check_err(bk_ctx* c) {
  int herr = 0;
  BK_CUDA(cudaMemcpy(&herr, c->d_err, sizeof(int), cudaMemcpyDeviceToHost));
  if (herr & kErrStageOverflow) return fail(BK_E_RANGE, "staged chunk exceeded its slot (internal bound violated)");
  if (herr & kErrKeyRange) return fail(BK_E_INVAL, "a group-by key is >= G");
  if (herr & kErrTableFull) return fail(BK_E_CAPACITY, "word-count hash table full; raise table_slots");
  if (herr & kErrWordTooLong) return fail(BK_E_RANGE, "a word is longer than 2^24 bytes or offset >= 2^40");
  return BK_OK;
}

// ---- the pipeline driver: chunk i goes through slot i % N; stages 1-3 on the copy/assembly
// streams, stage 4 on the compute stream. `concurrent`: the kernel's updates commute (atomic
// aggregation), so chunk i's compute runs on slot stream i % N and may overlap chunk i-1's;
// otherwise (grep's ordered output) every compute is serialised on s_comp.
template <class Compute>
int pipeline(bk_ctx* c, const Plan& p, bool concurrent, Compute&& compute) {
  const size_t C = p.bounds.size() - 1;
  c->st.n_chunks = C;
  note_plan(c, p);
  std::vector<cudaEvent_t> zc_inflight;
  const size_t zc_depth = std::max<size_t>(1, (c->cfg.n_slots - 1) / 2);
  if (p.mode == BK_GATHER_CPU || p.mode == BK_GATHER_HYBRID) {
    int rc = ensure_host_side(c, p);
    if (rc) return rc;
  }
  for (size_t i = 0; i < C; ++i) {
    Slot& s = c->slots[i % c->cfg.n_slots];
    cudaStream_t cs = concurrent ? c->s_slot[i % c->cfg.n_slots] : c->s_comp;
    bool cpu = p.mode == BK_GATHER_CPU;
    if (p.mode == BK_GATHER_HYBRID && c->cfg.zc_share_pm) {
      // deterministic split (profiling, reproducibility): chunk i is zero-copy iff
      // floor((i+1) s) > floor(i s)
      const uint64_t pm = std::min<uint32_t>(c->cfg.zc_share_pm, 1000);
      cpu = ((i + 1) * pm) / 1000 == (i * pm) / 1000;
    } else if (p.mode == BK_GATHER_HYBRID) {
      // adaptive split (default): the GPU zero-copy gathers run asynchronously; keep one in flight
      // and let the host pool assemble the next chunk while it is busy (profiles/r01_hybrid_sweep.md)
      while (!zc_inflight.empty() && cudaEventQuery(zc_inflight.front()) == cudaSuccess)
        zc_inflight.erase(zc_inflight.begin());
      cudaGetLastError();
      cpu = zc_inflight.size() >= zc_depth;
    }
    int rc = cpu ? stage_chunk_cpu(c, p, i, s) : stage_chunk(c, p, i, s);
    if (rc) return rc;
    if (p.mode == BK_GATHER_HYBRID && !cpu) zc_inflight.push_back(s.ready);
    BK_CUDA(cudaStreamWaitEvent(cs, s.ready, 0));
    BK_DELAY(cs);
    BK_PROF(kStCompute, cs, true);
    cudaStream_t rel = cs;   // stream whose completion frees the slot (partition: its D2H)
    rc = compute(chunk_of(c, p, i), s, cs, rel);
    if (rc) return rc;
    BK_PROF(kStCompute, cs, false);
    BK_CUDA(cudaEventRecord(s.freed, rel));
  }
  if (concurrent)  // join: finalize on s_comp after every slot's last compute
    for (auto& s : c->slots)
      if (s.used) BK_CUDA(cudaStreamWaitEvent(c->s_comp, s.freed, 0));
  return BK_OK;
}

Access whole_access() {
  Access a{};
  a.whole = 1;
  return a;
}
Access field_access(uint32_t off, uint32_t len) {
  Access a{};
  a.whole = 0;
  a.n_ext = 1;
  a.ext_off[0] = off;
  a.ext_len[0] = len;
  a.E = len;
  return a;
}

int begin_run(bk_ctx* c, void* stream) {
  BK_CUDA(cudaSetDevice(c->cfg.device));
  BK_CUDA(cudaMemsetAsync(c->d_err, 0, sizeof(int), c->s_comp));
  BK_CUDA(cudaMemsetAsync(c->d_ctr, 0, 8 * sizeof(unsigned long long), c->s_comp));
  BK_CUDA(cudaEventRecord(c->ev_begin, (cudaStream_t)stream));
  BK_CUDA(cudaStreamWaitEvent(c->s_comp, c->ev_begin, 0));
  BK_CUDA(cudaEventRecord(c->t_begin, c->s_comp));
  BK_CUDA(cudaEventRecord(c->ev_begin, c->s_comp));
  BK_CUDA(cudaStreamWaitEvent(c->s_copy, c->ev_begin, 0));
  BK_CUDA(cudaStreamWaitEvent(c->s_asm, c->ev_begin, 0));
  for (auto& s : c->slots) s.used = false;
  c->n_launch = 0;
  c->prof_used = 0;
  c->st.bytes_accessed = c->st.bytes_h2d = c->st.bytes_meta = c->st.bytes_padding = c->st.bytes_d2h = 0;
  c->st.n_chunks_cpu = 0;
  c->st.ms_cpu_gather = 0;
  return BK_OK;
}

// Per-stage busy sums and, from the interval of every (stage, chunk) event pair relative to the
// run start, the union of transfer intervals, the union of compute intervals and their overlap
// (the north_star's copy/compute overlap, measured with CUDA events instead of nsys).
int stage_stats(bk_ctx* c) {
  double acc[kNStages] = {0, 0, 0, 0, 0};
  uint64_t cnt[kNStages] = {0, 0, 0, 0, 0};
  std::vector<std::pair<double, double>> xfer, comp;
  for (size_t i = 0; i + 1 < c->prof_used + 1 && i < c->prof_used; i += 2) {
    float e = 0, b0 = 0;
    BK_CUDA(cudaEventElapsedTime(&e, c->prof[i], c->prof[i + 1]));
    BK_CUDA(cudaEventElapsedTime(&b0, c->t_begin, c->prof[i]));
    const int stg = c->prof_stage[i / 2];
    acc[stg] += e;
    cnt[stg] += 1;
    if (stg == kStH2D || stg == kStGather) xfer.emplace_back(b0, b0 + e);
    if (stg == kStCompute) comp.emplace_back(b0, b0 + e);
  }
  auto merge = [](std::vector<std::pair<double, double>> v) {
    std::sort(v.begin(), v.end());
    std::vector<std::pair<double, double>> u;
    for (auto& x : v) {
      if (!u.empty() && x.first <= u.back().second) u.back().second = std::max(u.back().second, x.second);
      else u.push_back(x);
    }
    return u;
  };
  const auto ux = merge(xfer), uc = merge(comp);
  double bx = 0, bc = 0, ov = 0;
  for (auto& x : ux) bx += x.second - x.first;
  for (auto& x : uc) bc += x.second - x.first;
  for (size_t i = 0, j = 0; i < ux.size() && j < uc.size();) {  // intersection of two sorted unions
    const double lo = std::max(ux[i].first, uc[j].first), hi = std::min(ux[i].second, uc[j].second);
    if (hi > lo) ov += hi - lo;
    if (ux[i].second < uc[j].second) ++i; else ++j;
  }
  c->st.ms_h2d = acc[kStH2D];
  c->st.ms_addrgen = acc[kStAddrgen];
  c->st.ms_gather = acc[kStGather] + acc[kStRelayout];
  c->st.ms_compute = acc[kStCompute];
  c->st.n_gather = cnt[kStGather] + cnt[kStRelayout];
  c->st.ms_xfer_busy = bx;
  c->st.ms_compute_busy = bc;
  c->st.ms_overlap = ov;
  return BK_OK;
}

int end_run(bk_ctx* c, void* stream) {
  BK_CUDA(cudaEventRecord(c->t_end, c->s_comp));
  BK_CUDA(cudaEventRecord(c->ev_end, c->s_comp));
  BK_CUDA(cudaStreamWaitEvent((cudaStream_t)stream, c->ev_end, 0));
  BK_CUDA(cudaStreamSynchronize(c->s_comp));
  unsigned long long staged = 0;
  BK_CUDA(cudaMemcpy(&staged, c->d_ctr + 0, 8, cudaMemcpyDeviceToHost));
  c->st.bytes_padding = staged >= c->st.bytes_accessed ? staged - c->st.bytes_accessed : 0;
  float ms = 0;
  BK_CUDA(cudaEventElapsedTime(&ms, c->t_begin, c->t_end));
  c->st.ms_device = ms;
  int rc = stage_stats(c);
  if (rc) return rc;
  return check_err(c);
}

// ---- run_device: fork/join all streams around a pipeline; capture it as a CUDA graph once per key
std::vector<cudaStream_t> side_streams(bk_ctx* c) {
  std::vector<cudaStream_t> v{c->s_copy, c->s_asm, c->s_d2h};
  for (auto st : c->s_slot) v.push_back(st);
  return v;
}

int device_begin(bk_ctx* c) {
  BK_CUDA(cudaMemsetAsync(c->d_err, 0, sizeof(int), c->s_comp));
  BK_CUDA(cudaMemsetAsync(c->d_ctr, 0, 8 * sizeof(unsigned long long), c->s_comp));
  BK_CUDA(cudaEventRecord(c->ev_fork, c->s_comp));
  for (auto st : side_streams(c)) BK_CUDA(cudaStreamWaitEvent(st, c->ev_fork, 0));
  return BK_OK;
}

int device_end(bk_ctx* c) {
  const auto ss = side_streams(c);
  for (size_t i = 0; i < ss.size(); ++i) {
    BK_CUDA(cudaEventRecord(c->ev_join[i], ss[i]));
    BK_CUDA(cudaStreamWaitEvent(c->s_comp, c->ev_join[i], 0));
  }
  return BK_OK;
}

void host_reset(bk_ctx* c) {
  for (auto& s : c->slots) s.used = false;
  c->n_launch = 0;
  c->prof_used = 0;
  c->st.bytes_accessed = c->st.bytes_h2d = c->st.bytes_meta = c->st.bytes_padding = c->st.bytes_d2h = 0;
  c->st.n_chunks_cpu = 0;
  c->st.ms_cpu_gather = 0;
}

int prof_reserve(bk_ctx* c, size_t pairs) {
  if (!(c->cfg.flags & BK_FLAG_PROFILE)) return BK_OK;
  while (c->prof.size() < 2 * pairs) {
    cudaEvent_t e;
    BK_CUDA(cudaEventCreate(&e));
    c->prof.push_back(e);
    if (c->prof.size() % 2 == 0) c->prof_stage.push_back(0);
  }
  return BK_OK;
}

int end_host(bk_ctx* c, void* stream) {
  BK_CUDA(cudaEventRecord(c->t_end, c->s_comp));   // outside any graph: graph event nodes carry no timestamps
  BK_CUDA(cudaEventRecord(c->ev_end, c->s_comp));
  BK_CUDA(cudaStreamWaitEvent((cudaStream_t)stream, c->ev_end, 0));
  BK_CUDA(cudaStreamSynchronize(c->s_comp));
  unsigned long long staged = 0;
  BK_CUDA(cudaMemcpy(&staged, c->d_ctr + 0, 8, cudaMemcpyDeviceToHost));
  c->st.bytes_padding = staged >= c->st.bytes_accessed ? staged - c->st.bytes_accessed : 0;
  float ms = 0;
  BK_CUDA(cudaEventElapsedTime(&ms, c->t_begin, c->t_end));
  c->st.ms_device = ms;
  int rc = stage_stats(c);
  if (rc) return rc;
  return check_err(c);
}

// Runs `enqueue` (which issues one whole pipeline on the context's streams) ordered after `stream`.
// ZC / DENSE pipelines are fully static for a given key, so the first run captures them as a
// CUDA graph and later runs replay it (BK_FLAG_NO_GRAPH forces eager issue).
template <class Enqueue>
int run_device(bk_ctx* c, void* stream, const std::string& key, bool graphable, size_t n_chunks, Enqueue&& enqueue) {
  BK_CUDA(cudaSetDevice(c->cfg.device));
  host_reset(c);
  BK_CUDA(cudaEventRecord(c->ev_begin, (cudaStream_t)stream));
  BK_CUDA(cudaStreamWaitEvent(c->s_comp, c->ev_begin, 0));
  BK_CUDA(cudaEventRecord(c->t_begin, c->s_comp));
  int rc;
  // per-stage profiling events must be real stream events (timestamps), so BK_FLAG_PROFILE issues eagerly
  if (!graphable || (c->cfg.flags & (BK_FLAG_NO_GRAPH | BK_FLAG_PROFILE))) {
    if ((rc = device_begin(c)) || (rc = enqueue()) || (rc = device_end(c))) return rc;
    return end_host(c, stream);
  }
  GraphEntry* ge = nullptr;
  for (auto& g : c->graphs)
    if (g.key == key) ge = &g;
  if (ge) {
    const double reg = c->st.ms_register;
    c->st = ge->st;
    c->st.ms_register = reg;
    c->n_launch = ge->n_launch;
    c->prof_used = ge->prof_used;
    for (size_t i = 0; i < ge->prof_stage.size(); ++i) c->prof_stage[i] = ge->prof_stage[i];
  } else {
    if ((rc = prof_reserve(c, 4 * n_chunks + 8))) return rc;
    BK_CUDA(cudaStreamBeginCapture(c->s_comp, cudaStreamCaptureModeThreadLocal));
    rc = device_begin(c);
    if (!rc) rc = enqueue();
    if (!rc) rc = device_end(c);
    cudaGraph_t graph = nullptr;
    const cudaError_t e = cudaStreamEndCapture(c->s_comp, &graph);
    if (rc) {
      if (graph) cudaGraphDestroy(graph);
      cudaGetLastError();
      return rc;
    }
    if (e != cudaSuccess) return fail(BK_E_CUDA, "graph capture: %s", cudaGetErrorString(e));
    GraphEntry g;
    g.key = key;
    const cudaError_t ie = cudaGraphInstantiate(&g.exec, graph, 0);
    cudaGraphDestroy(graph);
    if (ie != cudaSuccess) return fail(BK_E_CUDA, "cudaGraphInstantiate: %s", cudaGetErrorString(ie));
    g.st = c->st;
    g.n_launch = c->n_launch;
    g.prof_used = c->prof_used;
    g.prof_stage.assign(c->prof_stage.begin(), c->prof_stage.begin() + std::min(c->prof_stage.size(), c->prof_used / 2));
    c->graphs.push_back(std::move(g));
    ge = &c->graphs.back();
  }
  BK_CUDA(cudaGraphLaunch(ge->exec, c->s_comp));
  return end_host(c, stream);
}

void drop_graphs(bk_ctx* c) {
  for (auto& g : c->graphs)
    if (g.exec) cudaGraphExecDestroy(g.exec);
  c->graphs.clear();
}

bool graphable(const Plan& p) { return p.mode == BK_GATHER_ZC || p.mode == BK_GATHER_DENSE; }

// ------------------------------------------------------------------ kernels
int run_wordcount(bk_ctx* c, bk_out_wordcount* o, void* stream) {
  uint64_t slots = o->table_slots ? o->table_slots : (1ull << 20);
  if (slots & (slots - 1)) return fail(BK_E_INVAL, "table_slots must be a power of two");
  Plan p;
  // word count is compute-bound (thread-per-lane scan + table updates): AUTO picks ZC, which needs
  // no raw buffer, so the window holds twice the text in flight; 256-B lanes (profiles/r01_wc_sweep.md)
  int rc = plan_run(c, whole_access(), 256, p, 0, BK_GATHER_ZC);
  if (rc) return rc;
  carve(c, p);
  BK_CUDA(c->b_table.ensure(slots * sizeof(WcEntry)));
  const uint64_t ocap = std::min<uint64_t>(o->cap, slots);
  BK_CUDA(c->b_out1.ensure(std::max<uint64_t>(ocap, 1) * 8));
  BK_CUDA(c->b_out2.ensure(std::max<uint64_t>(ocap, 1) * 4));
  BK_CUDA(c->b_out3.ensure(std::max<uint64_t>(ocap, 1) * 8));
  WcEntry* table = (WcEntry*)c->b_table.p;
  const std::string key = "wc/" + std::to_string(slots) + "/" + std::to_string(ocap) + "/" + p.key;
  rc = run_device(c, stream, key, graphable(p), p.bounds.size() - 1, [&]() -> int {
    BK_CUDA(cudaMemsetAsync(c->b_table.p, 0, slots * sizeof(WcEntry), c->s_comp));
    int r = pipeline(c, p, true, [&](const Chunk& ch, Slot& s, cudaStream_t cs, cudaStream_t&) {
      launch_wc(ch, s.stage, s.lanes, s.tile_base, s.meta, c->off ? 0 : c->cfg.record_size, table, slots - 1,
                c->d_ctr + 1, c->d_err, cs);
      c->n_launch += 1;
      return BK_OK;
    });
    if (r) return r;
    launch_wc_compact(table, slots, c->d_ctr + 2, (uint64_t*)c->b_out1.p, (uint32_t*)c->b_out2.p,
                      (uint64_t*)c->b_out3.p, ocap, c->s_comp);
    c->n_launch += 1;
    return (int)BK_OK;
  });
  if (rc) return rc;
  unsigned long long nw = 0;
  BK_CUDA(cudaMemcpy(&nw, c->d_ctr + 2, 8, cudaMemcpyDeviceToHost));
  o->n_words = nw;
  if (nw > o->cap) return fail(BK_E_CAPACITY, "%llu distinct words > cap %llu", nw, (unsigned long long)o->cap);
  if (nw * 2 > slots) return fail(BK_E_CAPACITY, "table load %llu/%llu too high; raise table_slots", nw,
                                  (unsigned long long)slots);
  if (nw) {
    BK_CUDA(cudaMemcpy(o->word_off, c->b_out1.p, nw * 8, cudaMemcpyDeviceToHost));
    BK_CUDA(cudaMemcpy(o->word_len, c->b_out2.p, nw * 4, cudaMemcpyDeviceToHost));
    BK_CUDA(cudaMemcpy(o->word_count, c->b_out3.p, nw * 8, cudaMemcpyDeviceToHost));
  }
  uint64_t tot = 0;
  for (uint64_t i = 0; i < nw; ++i) tot += o->word_count[i];
  o->total_words = tot;
  c->st.bytes_d2h = nw * 20;
  return BK_OK;
}

int run_grep(bk_ctx* c, bk_out_grep* o, void* stream) {
  if (o->pattern_len > 32) return fail(BK_E_INVAL, "pattern longer than 32 bytes");
  if (o->pattern_len && !o->pattern) return fail(BK_E_INVAL, "NULL pattern");
  if (c->min_rec < 48) return fail(BK_E_INVAL, "grep needs records of >= 48 bytes (key at +16..+48)");
  Plan p;
  int rc = plan_run(c, field_access(16, 32), 256, p);
  if (rc) return rc;
  carve(c, p);
  const uint32_t nblk = (p.L + 255) / 256;
  const uint64_t cap = std::min<uint64_t>(o->cap, c->n);
  BK_CUDA(c->b_out1.ensure(std::max<uint64_t>(cap, 1) * 8));
  BK_CUDA(c->b_blk.ensure((uint64_t)nblk * 4));
  BK_CUDA(c->b_blk2.ensure((uint64_t)nblk * 8));
  GrepParams gp{};
  if (o->pattern_len) memcpy(gp.pat, o->pattern, o->pattern_len);
  gp.plen = o->pattern_len;
  gp.first_index = o->first_index;
  gp.cap = cap;
  std::string key = "grep/" + std::to_string(gp.plen) + "/" + std::to_string(gp.first_index) + "/" +
                    std::to_string(gp.cap) + "/" + p.key + "/";
  for (uint32_t i = 0; i < gp.plen; ++i) key += std::to_string(gp.pat[i]) + ",";
  rc = run_device(c, stream, key, graphable(p), p.bounds.size() - 1, [&]() -> int {
    return pipeline(c, p, false, [&](const Chunk& ch, Slot& s, cudaStream_t cs, cudaStream_t&) {
      launch_grep(ch, s.stage, s.lanes, s.tile_base, gp, (uint32_t*)c->b_blk.p, c->d_ctr + 3,
                  (unsigned long long*)c->b_blk2.p, (uint64_t*)c->b_out1.p, c->d_err, cs);
      c->n_launch += 3;
      return BK_OK;
    });
  });
  if (rc) return rc;
  unsigned long long m = 0;
  BK_CUDA(cudaMemcpy(&m, c->d_ctr + 3, 8, cudaMemcpyDeviceToHost));
  o->n_match = m;
  if (m > o->cap) return fail(BK_E_CAPACITY, "%llu matches > cap %llu", m, (unsigned long long)o->cap);
  if (m) BK_CUDA(cudaMemcpy(o->idx, c->b_out1.p, m * 8, cudaMemcpyDeviceToHost));
  c->st.bytes_d2h = m * 8;
  return BK_OK;
}

int run_groupby(bk_ctx* c, bk_out_groupby* o, void* stream) {
  const uint32_t G = o->G;
  if (G == 0 || G > 8192) return fail(BK_E_INVAL, "G must be in 1..8192");
  if (c->min_rec < 16) return fail(BK_E_INVAL, "group-by records must be >= 16 bytes");
  const bool dense16 = !c->off && c->cfg.record_size == 16;
  Plan p;
  int rc = plan_run(c, dense16 ? whole_access() : field_access(0, 16), 256, p);
  if (rc) return rc;
  carve(c, p);
  BK_CUDA(c->b_agg1.ensure((uint64_t)G * 8));
  BK_CUDA(c->b_agg2.ensure((uint64_t)G * 8));
  BK_CUDA(c->b_agg3.ensure((uint64_t)G * 8));
  int dev_sms = 148, per_sm = 1;
  cudaDeviceGetAttribute(&dev_sms, cudaDevAttrMultiProcessorCount, c->cfg.device);
  per_sm = std::max<int>(1, (int)((200 * 1024) / std::max<size_t>(groupby_smem(G), 1)));
  per_sm = std::min(per_sm, 4);
  const int grid = std::max(1, std::min<int>((p.L + 255) / 256, dev_sms * per_sm));
  rc = run_device(c, stream, "groupby/" + std::to_string(G) + "/" + p.key, graphable(p), p.bounds.size() - 1,
                  [&]() -> int {
    BK_CUDA(cudaMemsetAsync(c->b_agg1.p, 0, (uint64_t)G * 8, c->s_comp));
    BK_CUDA(cudaMemsetAsync(c->b_agg2.p, 0, (uint64_t)G * 8, c->s_comp));
    BK_CUDA(cudaMemsetAsync(c->b_agg3.p, 0, (uint64_t)G * 8, c->s_comp));
    return pipeline(c, p, true, [&](const Chunk& ch, Slot& s, cudaStream_t cs, cudaStream_t&) {
      launch_groupby(ch, s.stage, s.lanes, s.tile_base, G, (unsigned long long*)c->b_agg1.p,
                     (unsigned long long*)c->b_agg2.p, (double*)c->b_agg3.p, c->d_err, grid, cs);
      c->n_launch += 1;
      return BK_OK;
    });
  });
  if (rc) return rc;
  BK_CUDA(cudaMemcpy(o->count, c->b_agg1.p, (uint64_t)G * 8, cudaMemcpyDeviceToHost));
  BK_CUDA(cudaMemcpy(o->qty, c->b_agg2.p, (uint64_t)G * 8, cudaMemcpyDeviceToHost));
  BK_CUDA(cudaMemcpy(o->amount, c->b_agg3.p, (uint64_t)G * 8, cudaMemcpyDeviceToHost));
  c->st.bytes_d2h = (uint64_t)G * 24;
  return BK_OK;
}

// The caller's per-record output (partition records, k-means cid) is written by DMA: pin it once
// and keep it pinned across runs (one cached registration per context).
int ensure_out_pinned(bk_ctx* c, void* ptr, uint64_t bytes) {
  if (!bytes) return BK_OK;
  for (auto& e : c->out_pinned)
    if (e.first == ptr && e.second == bytes) return BK_OK;
  if (is_pinned(ptr)) return BK_OK;
  if (c->out_pinned.size() >= 4) {  // keep at most four cached registrations (oldest out)
    cudaHostUnregister(c->out_pinned.front().first);
    c->out_pinned.erase(c->out_pinned.begin());
  }
  BK_CUDA(cudaHostRegister(ptr, bytes, cudaHostRegisterPortable));
  c->out_pinned.emplace_back(ptr, bytes);
  return BK_OK;
}

int run_kmeans(bk_ctx* c, bk_out_kmeans* o, void* stream) {
  const uint32_t K = o->K;
  if (K == 0 || K > 256 || !o->centroids) return fail(BK_E_INVAL, "K must be in 1..256 with centroids");
  if (c->min_rec < 64) return fail(BK_E_INVAL, "k-means records must hold 16 fp32 (>= 64 bytes)");
  const bool dense64 = !c->off && c->cfg.record_size == 64;
  Plan p;
  // cid write-back (P:563-572 writes to mapped data; "sets its clusterId"): 4 B per
  // record per chunk in the slot, DMA'd back on the D2H stream while the next chunks stream in
  int rc = plan_run(c, dense64 ? whole_access() : field_access(0, 64), 256, p, o->cid ? 4 : 0);
  if (rc) return rc;
  carve(c, p);
  if (o->cid && (rc = ensure_out_pinned(c, o->cid, c->n * 4))) return rc;
  BK_CUDA(c->b_mu.ensure((uint64_t)K * 64));
  BK_CUDA(c->b_agg1.ensure((uint64_t)K * 8));
  BK_CUDA(c->b_agg3.ensure((uint64_t)K * 16 * 8));
  int dev_sms = 148;
  cudaDeviceGetAttribute(&dev_sms, cudaDevAttrMultiProcessorCount, c->cfg.device);
  if (!c->h_mu) BK_CUDA(cudaHostAlloc((void**)&c->h_mu, 256 * 64, cudaHostAllocPortable));
  memcpy(c->h_mu, o->centroids, (size_t)K * 64);   // the graph copies from this pinned buffer
  const int grid = std::max(1, std::min<int>((p.L + 255) / 256, dev_sms * 2));
  const std::string key = "kmeans/" + std::to_string(K) + "/" + std::to_string(o->first_index) + "/" +
                          std::to_string((uintptr_t)o->cid) + "/" + p.key;
  rc = run_device(c, stream, key, graphable(p), p.bounds.size() - 1, [&]() -> int {
  BK_CUDA(cudaMemcpyAsync(c->b_mu.p, c->h_mu, (uint64_t)K * 64, cudaMemcpyHostToDevice, c->s_comp));
  BK_CUDA(cudaMemsetAsync(c->b_agg1.p, 0, (uint64_t)K * 8, c->s_comp));
  BK_CUDA(cudaMemsetAsync(c->b_agg3.p, 0, (uint64_t)K * 128, c->s_comp));
  size_t ci = 0;
  int r = pipeline(c, p, true, [&](const Chunk& ch, Slot& s, cudaStream_t cs, cudaStream_t& rel) -> int {
    launch_kmeans(ch, s.stage, s.lanes, s.tile_base, (const float*)c->b_mu.p, K, o->first_index,
                  (unsigned long long*)c->b_agg1.p, (double*)c->b_agg3.p, c->d_ctr + 4,
                  o->cid ? (int32_t*)s.out : nullptr, grid, cs);
    c->n_launch += 1;
    if (o->cid && ch.hi > ch.lo) {
      cudaEvent_t e = c->ev_part[ci++ % c->ev_part.size()];
      BK_CUDA(cudaEventRecord(e, cs));
      BK_CUDA(cudaStreamWaitEvent(c->s_d2h, e, 0));
      BK_CUDA(cudaMemcpyAsync(o->cid + ch.lo, s.out, (ch.hi - ch.lo) * 4, cudaMemcpyDeviceToHost, c->s_d2h));
      c->st.bytes_d2h += (ch.hi - ch.lo) * 4;
      rel = c->s_d2h;
    }
    return (int)BK_OK;
  });
  return r;
  });
  if (rc) return rc;
  BK_CUDA(cudaMemcpy(o->count, c->b_agg1.p, (uint64_t)K * 8, cudaMemcpyDeviceToHost));
  BK_CUDA(cudaMemcpy(o->sum, c->b_agg3.p, (uint64_t)K * 128, cudaMemcpyDeviceToHost));
  unsigned long long chk = 0;
  BK_CUDA(cudaMemcpy(&chk, c->d_ctr + 4, 8, cudaMemcpyDeviceToHost));
  o->chk = chk;
  c->st.bytes_d2h += (uint64_t)K * 136;
  return BK_OK;
}

// f4: k-mer counting (FIELD access to the sequence; the table is resident, outside the window)
int run_kmer(bk_ctx* c, bk_out_kmer* o, void* stream) {
  const uint64_t slots = o->table_slots ? o->table_slots : (1ull << 24);
  if (slots & (slots - 1)) return fail(BK_E_INVAL, "table_slots must be a power of two");
  if (o->k < 1 || o->k > 31) return fail(BK_E_INVAL, "k must be in 1..31");
  if (o->seq_len == 0 || o->seq_len % 16) return fail(BK_E_INVAL, "seq_len must be a positive multiple of 16");
  if ((uint64_t)o->seq_off + o->seq_len > c->min_rec) return fail(BK_E_INVAL, "sequence field exceeds a record");
  Plan p;
  int rc = plan_run(c, field_access(o->seq_off, o->seq_len), 256, p);
  if (rc) return rc;
  carve(c, p);
  BK_CUDA(c->b_table.ensure(slots * sizeof(KmerEntry)));
  const uint64_t ocap = std::min<uint64_t>(o->cap, slots);
  BK_CUDA(c->b_out1.ensure(std::max<uint64_t>(ocap, 1) * 8));
  BK_CUDA(c->b_out3.ensure(std::max<uint64_t>(ocap, 1) * 8));
  KmerEntry* table = (KmerEntry*)c->b_table.p;
  const std::string key = "kmer/" + std::to_string(o->k) + "/" + std::to_string(slots) + "/" + std::to_string(ocap) +
                          "/" + p.key;
  rc = run_device(c, stream, key, graphable(p), p.bounds.size() - 1, [&]() -> int {
    BK_CUDA(cudaMemsetAsync(c->b_table.p, 0, slots * sizeof(KmerEntry), c->s_comp));
    int r = pipeline(c, p, true, [&](const Chunk& ch, Slot& s, cudaStream_t cs, cudaStream_t&) {
      launch_kmer(ch, s.stage, s.lanes, s.tile_base, o->k, o->seq_len / 16, table, slots - 1, c->d_ctr + 1,
                  c->d_ctr + 5, c->d_err, cs);
      c->n_launch += 1;
      return BK_OK;
    });
    if (r) return r;
    launch_kmer_compact(table, slots, c->d_ctr + 2, (uint64_t*)c->b_out1.p, (uint64_t*)c->b_out3.p, ocap, c->s_comp);
    c->n_launch += 1;
    return (int)BK_OK;
  });
  if (rc) return rc;
  unsigned long long nk = 0, tot = 0;
  BK_CUDA(cudaMemcpy(&nk, c->d_ctr + 2, 8, cudaMemcpyDeviceToHost));
  BK_CUDA(cudaMemcpy(&tot, c->d_ctr + 5, 8, cudaMemcpyDeviceToHost));
  o->n_kmers = nk;
  o->total = tot;
  if (nk > o->cap) return fail(BK_E_CAPACITY, "%llu distinct k-mers > cap %llu", nk, (unsigned long long)o->cap);
  if (nk * 10 > slots * 7) return fail(BK_E_CAPACITY, "k-mer table load %llu/%llu too high; raise table_slots", nk,
                                       (unsigned long long)slots);
  if (nk) {
    // the result arrays are large (16 B per distinct k-mer): pin them once so the copy runs at DMA speed
    if ((rc = ensure_out_pinned(c, o->kmer, o->cap * 8)) || (rc = ensure_out_pinned(c, o->count, o->cap * 8))) return rc;
    BK_CUDA(cudaMemcpy(o->kmer, c->b_out1.p, nk * 8, cudaMemcpyDeviceToHost));
    BK_CUDA(cudaMemcpy(o->count, c->b_out3.p, nk * 8, cudaMemcpyDeviceToHost));
  }
  c->st.bytes_d2h = nk * 16;
  return BK_OK;
}

int run_partition(bk_ctx* c, bk_out_partition* o, void* stream) {
  const uint32_t B = o->n_buckets;
  if (B == 0 || B > 4096 || (B & (B - 1))) return fail(BK_E_INVAL, "n_buckets must be a power of two in 1..4096");
  if (c->off || c->cfg.record_size != 16) return fail(BK_E_INVAL, "partition needs fixed 16-byte {key, value} records");
  if (c->n && !o->out_records) return fail(BK_E_INVAL, "NULL out_records");
  int bits = 0;
  while ((1u << bits) < B) ++bits;
  Plan p;
  int rc = plan_run(c, whole_access(), 256, p, 16);
  if (rc) return rc;
  carve(c, p);
  const uint64_t C = p.bounds.size() - 1;
  o->n_chunks = C;
  if (C > o->chunk_cap) return fail(BK_E_CAPACITY, "%llu chunks > chunk_cap %llu", (unsigned long long)C,
                                    (unsigned long long)o->chunk_cap);
  uint32_t nblk_max = 1;
  for (uint64_t i = 0; i < C; ++i) nblk_max = std::max(nblk_max, partition_blocks(chunk_of(c, p, i)));
  BK_CUDA(c->b_hist.ensure((uint64_t)nblk_max * B * 4));
  BK_CUDA(c->b_colpre.ensure((uint64_t)nblk_max * B * 4));
  BK_CUDA(c->b_totals.ensure(std::max<uint64_t>(C, 1) * B * 8));
  BK_CUDA(c->b_base.ensure((uint64_t)B * 8));
  if ((rc = ensure_out_pinned(c, o->out_records, c->n * 16))) return rc;
  const std::string key = "part/" + std::to_string(B) + "/" + std::to_string((uintptr_t)o->out_records) + "/" + p.key;
  rc = run_device(c, stream, key, graphable(p), p.bounds.size() - 1, [&]() -> int {
  size_t ci = 0;
  return pipeline(c, p, false, [&](const Chunk& ch, Slot& s, cudaStream_t cs, cudaStream_t& rel) -> int {
    launch_partition(ch, s.stage, s.lanes, s.tile_base, bits, (uint32_t*)c->b_hist.p, (uint32_t*)c->b_colpre.p,
                     (unsigned long long*)c->b_totals.p + ci * B, (unsigned long long*)c->b_base.p, s.out, cs);
    c->n_launch += 4;
    cudaEvent_t e = c->ev_part[ci % c->ev_part.size()];
    BK_CUDA(cudaEventRecord(e, cs));
    BK_CUDA(cudaStreamWaitEvent(c->s_d2h, e, 0));
    const uint64_t bytes = (ch.hi - ch.lo) * 16;
    if (bytes)
      BK_CUDA(cudaMemcpyAsync((uint8_t*)o->out_records + ch.lo * 16, s.out, bytes, cudaMemcpyDeviceToHost, c->s_d2h));
    c->st.bytes_d2h += bytes;
    rel = c->s_d2h;
    ++ci;
    return (int)BK_OK;
  });
  });
  if (rc) return rc;
  std::vector<uint64_t> tot(C * B);
  if (C) BK_CUDA(cudaMemcpy(tot.data(), c->b_totals.p, C * B * 8, cudaMemcpyDeviceToHost));
  for (uint32_t b = 0; b < B; ++b) o->bucket_count[b] = 0;
  for (uint64_t i = 0; i < C; ++i)
    for (uint32_t b = 0; b < B; ++b) {
      o->chunk_counts[i * B + b] = tot[i * B + b];
      o->bucket_count[b] += tot[i * B + b];
    }
  return BK_OK;
}

// ---- BK_FLAG_BASELINE_DBUF: the traditional chunked loop with two buffers ----
int run_dbuf(bk_ctx* c, int kid, void* out, void* stream) {
  if (kid != BK_K_GREP && kid != BK_K_GROUPBY) return fail(BK_E_UNSUPPORTED, "dbuf baseline: grep / group-by only");
  Plan p;
  p.a = whole_access();
  p.mode = BK_GATHER_DENSE;
  p.zero_copy = 0;
  const bool single = (c->cfg.flags & BK_FLAG_BASELINE_SBUF) != 0;
  const uint64_t half = c->cfg.window_bytes / (single ? 1 : 2) / kAlign * kAlign;
  uint64_t budget = std::max<uint64_t>(std::min<uint64_t>(half, std::max<uint64_t>(c->nbytes / 32, 1ull << 20)), 1);
  uint64_t meta_cap = 0;
  for (int it = 0;; ++it) {
    p.budget = budget;
    int rc = make_chunks(c, p);
    if (rc) return rc;
    uint64_t maxrecs = 0;
    for (size_t i = 0; i + 1 < p.bounds.size(); ++i) maxrecs = std::max<uint64_t>(maxrecs, p.bounds[i + 1] - p.bounds[i]);
    meta_cap = c->off ? maxrecs + 1 : 0;
    if (align_up(budget + 64, kAlign) + meta_cap * 8 <= half) break;
    if (it > 64 || budget < 64) return fail(BK_E_NOMEM, "window too small for the dbuf baseline");
    budget = budget * 3 / 4;
  }
  uint8_t* buf[2] = {c->window, c->window + (single ? 0 : half)};
  uint64_t* meta[2] = {reinterpret_cast<uint64_t*>(buf[0] + align_up(budget + 64, kAlign)),
                       reinterpret_cast<uint64_t*>(buf[1] + align_up(budget + 64, kAlign))};
  cudaStream_t sb[2] = {c->s_copy, single ? c->s_copy : c->s_asm};
  const size_t C = p.bounds.size() - 1;
  int rc;
  GrepParams gp{};
  bk_out_grep* og = (bk_out_grep*)out;
  bk_out_groupby* ob = (bk_out_groupby*)out;
  const uint32_t nb = dbuf_blocks();
  if (kid == BK_K_GREP) {
    if (og->pattern_len > 32) return fail(BK_E_INVAL, "pattern longer than 32 bytes");
    if (c->min_rec < 48) return fail(BK_E_INVAL, "grep needs records of >= 48 bytes");
    if (og->pattern_len) memcpy(gp.pat, og->pattern, og->pattern_len);
    gp.plen = og->pattern_len;
    gp.first_index = og->first_index;
    gp.cap = std::min<uint64_t>(og->cap, c->n);
    BK_CUDA(c->b_out1.ensure(std::max<uint64_t>(gp.cap, 1) * 8));
    BK_CUDA(c->b_blk.ensure((uint64_t)nb * 4 * 2));
    BK_CUDA(c->b_blk2.ensure((uint64_t)nb * 8 * 2));
  } else {
    if (ob->G == 0 || ob->G > 8192) return fail(BK_E_INVAL, "G must be in 1..8192");
    if (c->off || c->cfg.record_size < 16) return fail(BK_E_INVAL, "group-by needs fixed records >= 16 B");
    BK_CUDA(c->b_agg1.ensure((uint64_t)ob->G * 8));
    BK_CUDA(c->b_agg2.ensure((uint64_t)ob->G * 8));
    BK_CUDA(c->b_agg3.ensure((uint64_t)ob->G * 8));
  }
  if ((rc = begin_run(c, stream))) return rc;
  if (kid == BK_K_GROUPBY) {
    BK_CUDA(cudaMemsetAsync(c->b_agg1.p, 0, (uint64_t)ob->G * 8, c->s_comp));
    BK_CUDA(cudaMemsetAsync(c->b_agg2.p, 0, (uint64_t)ob->G * 8, c->s_comp));
    BK_CUDA(cudaMemsetAsync(c->b_agg3.p, 0, (uint64_t)ob->G * 8, c->s_comp));
    BK_CUDA(cudaEventRecord(c->ev_begin, c->s_comp));
    BK_CUDA(cudaStreamWaitEvent(c->s_copy, c->ev_begin, 0));
    BK_CUDA(cudaStreamWaitEvent(c->s_asm, c->ev_begin, 0));
  }
  c->st.n_chunks = C;
  c->st.gather_mode = BK_GATHER_DENSE;
  c->st.chunk_budget = budget;
  cudaEvent_t scanned[2] = {c->slots[0].ready, c->slots[1].ready};
  for (size_t i = 0; i < C; ++i) {
    const int b = (int)(i & 1);
    cudaStream_t st = sb[b];
    const uint64_t lo = p.bounds[i], hi = p.bounds[i + 1];
    const uint64_t base = rec_start(c, lo), end = rec_start(c, hi);
    const uint64_t raw_off = ((uintptr_t)(c->host + base)) & 15;
    BK_PROF(kStH2D, st, true);
    if (end > base) BK_CUDA(cudaMemcpyAsync(buf[b] + raw_off, c->host + base, end - base, cudaMemcpyHostToDevice, st));
    if (c->off && hi > lo) {
      BK_CUDA(cudaMemcpyAsync(meta[b], c->off + lo, (hi - lo) * 8, cudaMemcpyHostToDevice, st));
      c->st.bytes_meta += (hi - lo) * 8;
    }
    BK_PROF(kStH2D, st, false);
    c->st.bytes_h2d += end - base;
    BK_PROF(kStCompute, st, true);
    if (kid == BK_K_GREP) {
      // chunk i's output offset follows chunk i-1's scan (ordered results across the two streams)
      if (i > 0) BK_CUDA(cudaStreamWaitEvent(st, scanned[1 - b], 0));
      launch_dbuf_grep(buf[b] + raw_off, c->off ? meta[b] : nullptr, lo, hi, base, end, c->cfg.record_size, gp,
                       (uint32_t*)c->b_blk.p + b * nb, c->d_ctr + 3, (unsigned long long*)c->b_blk2.p + b * nb,
                       (uint64_t*)c->b_out1.p, st);
      BK_CUDA(cudaEventRecord(scanned[b], st));
      c->n_launch += 3;
    } else {
      launch_dbuf_groupby(buf[b] + raw_off, lo, hi, base, c->cfg.record_size, ob->G, (unsigned long long*)c->b_agg1.p,
                          (unsigned long long*)c->b_agg2.p, (double*)c->b_agg3.p, c->d_err, st);
      c->n_launch += 1;
    }
    BK_PROF(kStCompute, st, false);
  }
  for (cudaStream_t st : sb) {
    BK_CUDA(cudaEventRecord(c->ev_end, st));
    BK_CUDA(cudaStreamWaitEvent(c->s_comp, c->ev_end, 0));
  }
  if ((rc = end_run(c, stream))) return rc;
  if (kid == BK_K_GREP) {
    unsigned long long m = 0;
    BK_CUDA(cudaMemcpy(&m, c->d_ctr + 3, 8, cudaMemcpyDeviceToHost));
    og->n_match = m;
    if (m > og->cap) return fail(BK_E_CAPACITY, "%llu matches > cap %llu", m, (unsigned long long)og->cap);
    if (m) BK_CUDA(cudaMemcpy(og->idx, c->b_out1.p, m * 8, cudaMemcpyDeviceToHost));
  } else {
    BK_CUDA(cudaMemcpy(ob->count, c->b_agg1.p, (uint64_t)ob->G * 8, cudaMemcpyDeviceToHost));
    BK_CUDA(cudaMemcpy(ob->qty, c->b_agg2.p, (uint64_t)ob->G * 8, cudaMemcpyDeviceToHost));
    BK_CUDA(cudaMemcpy(ob->amount, c->b_agg3.p, (uint64_t)ob->G * 8, cudaMemcpyDeviceToHost));
  }
  return BK_OK;
}

// caller-given access spec (test / experiment kernels): n_ext == 0 = whole record
int parse_access(const bk_ctx* c, uint32_t n_ext, const uint32_t* eo, const uint32_t* el, Access& a) {
  a = Access{};
  if (n_ext == 0) {
    a = whole_access();
    return BK_OK;
  }
  if (n_ext > (uint32_t)kMaxExt) return fail(BK_E_INVAL, "n_ext > %d", kMaxExt);
  a.n_ext = n_ext;
  for (uint32_t e = 0; e < n_ext; ++e) {
    a.ext_off[e] = eo[e];
    a.ext_len[e] = el[e];
    a.E += el[e];
    if ((uint64_t)eo[e] + el[e] > c->min_rec) return fail(BK_E_INVAL, "extent %u exceeds the shortest record", e);
  }
  return BK_OK;
}

// BK_K_PATTERN_STATS: stage 1 in address mode with online pattern recognition, every chunk
int run_pattern(bk_ctx* c, bk_out_pattern* o, void* stream) {
  Access a;
  int rc = parse_access(c, o->n_ext, o->ext_off, o->ext_len, a);
  if (rc) return rc;
  if (o->elem_bytes == 0 || o->T < 2 || o->T > 16 || o->pmax < 1 || o->pmax > 4)
    return fail(BK_E_INVAL, "elem_bytes >= 1, T in 2..16, pmax in 1..4");
  Plan p;
  if ((rc = plan_run(c, a, 256, p))) return rc;
  carve(c, p);
  a.rec_size = c->off ? 0 : c->cfg.record_size;
  o->lanes = p.L;
  const bool want_dump = o->chunk != UINT64_MAX;
  if (want_dump && (o->chunk >= p.bounds.size() - 1 || p.L > o->lane_cap))
    return fail(BK_E_INVAL, "dump chunk / lane_cap");
  BK_CUDA(c->b_out1.ensure((uint64_t)p.L * 4));
  BK_CUDA(c->b_out2.ensure((uint64_t)p.L * 32));
  BK_CUDA(c->b_out3.ensure((uint64_t)p.L * 16));
  BK_CUDA(c->b_blk2.ensure(8 * 8));
  if ((rc = begin_run(c, stream))) return rc;
  BK_CUDA(cudaMemsetAsync(c->b_blk2.p, 0, 64, c->s_copy));
  Slot& s = c->slots[0];
  for (size_t i = 0; i + 1 < p.bounds.size(); ++i) {  // one stream, one slot: stage 1 only
    const Chunk ch = chunk_of(c, p, i);
    if (c->off && ch.hi > ch.lo)
      BK_CUDA(cudaMemcpyAsync(s.meta, c->off + ch.lo, (ch.hi - ch.lo) * 8, cudaMemcpyHostToDevice, c->s_copy));
    launch_addrgen(ch, a, s.meta, s.lanes, s.tileK, s.tile_base, p.stage_cap, c->d_err, c->d_ctr + 0, c->s_copy);
    uint64_t* dumps = (uint64_t*)c->b_out3.p;
    launch_addr_patterns(ch, a, s.meta, s.lanes, o->elem_bytes, o->T, o->pmax, (int32_t*)c->b_out1.p,
                         (int64_t*)c->b_out2.p, dumps, dumps + p.L, (unsigned long long*)c->b_blk2.p,
                         want_dump && i == o->chunk, c->s_copy);
    c->n_launch += 3;
  }
  BK_CUDA(cudaEventRecord(c->ev_end, c->s_copy));
  BK_CUDA(cudaStreamWaitEvent(c->s_comp, c->ev_end, 0));
  if ((rc = end_run(c, stream))) return rc;
  unsigned long long tot[5];
  BK_CUDA(cudaMemcpy(tot, c->b_blk2.p, sizeof tot, cudaMemcpyDeviceToHost));
  o->n_lanes = tot[0];
  o->n_pattern_lanes = tot[1];
  o->n_addresses = tot[2];
  o->n_explicit_addresses = tot[3];
  o->address_bytes = 8 * tot[2];
  o->pattern_bytes = tot[4] + 8 * tot[3];
  if (want_dump) {
    BK_CUDA(cudaMemcpy(o->lane_p, c->b_out1.p, (uint64_t)p.L * 4, cudaMemcpyDeviceToHost));
    BK_CUDA(cudaMemcpy(o->lane_strides, c->b_out2.p, (uint64_t)p.L * 32, cudaMemcpyDeviceToHost));
    BK_CUDA(cudaMemcpy(o->lane_base, c->b_out3.p, (uint64_t)p.L * 8, cudaMemcpyDeviceToHost));
    BK_CUDA(cudaMemcpy(o->lane_count, (uint64_t*)c->b_out3.p + p.L, (uint64_t)p.L * 8, cudaMemcpyDeviceToHost));
  }
  return BK_OK;
}

int run_layout(bk_ctx* c, bk_out_layout* o, void* stream) {
  Access a;
  int rc = parse_access(c, o->n_ext, o->ext_off, o->ext_len, a);
  if (rc) return rc;
  Plan p;
  rc = plan_run(c, a, 256, p);
  if (rc) return rc;
  carve(c, p);
  o->n_chunks = p.bounds.size() - 1;
  o->lanes = p.L;
  if (o->chunk >= o->n_chunks) return fail(BK_E_INVAL, "chunk %llu >= %llu chunks", (unsigned long long)o->chunk,
                                           (unsigned long long)o->n_chunks);
  if ((rc = begin_run(c, stream))) return rc;
  Slot& s = c->slots[0];
  if (p.mode == BK_GATHER_CPU || p.mode == BK_GATHER_HYBRID) {
    if ((rc = ensure_host_side(c, p))) return rc;
    if ((rc = stage_chunk_cpu(c, p, o->chunk, s))) return rc;
  } else if ((rc = stage_chunk(c, p, o->chunk, s))) {
    return rc;
  }
  BK_CUDA(cudaStreamWaitEvent(c->s_comp, s.ready, 0));
  const Chunk ch = chunk_of(c, p, o->chunk);
  o->chunk_lo = ch.lo;
  o->chunk_hi = ch.hi;
  if ((rc = end_run(c, stream))) return rc;
  uint64_t size = 0;
  BK_CUDA(cudaMemcpy(&size, s.tile_base + ch.ntiles, 8, cudaMemcpyDeviceToHost));
  o->stage_size = size;
  if (size > o->stage_cap || p.L > o->lane_cap) return fail(BK_E_CAPACITY, "stage %llu / lanes %u", size, p.L);
  BK_CUDA(cudaMemcpy(o->stage, s.stage, size, cudaMemcpyDeviceToHost));
  std::vector<LaneDesc> ld(p.L);
  BK_CUDA(cudaMemcpy(ld.data(), s.lanes, (uint64_t)p.L * sizeof(LaneDesc), cudaMemcpyDeviceToHost));
  for (uint32_t t = 0; t < p.L; ++t) {
    o->lane_first[t] = ld[t].first;
    o->lane_nrec[t] = ld[t].nrec;
    o->lane_bytes[t] = ld[t].nbytes;
  }
  return BK_OK;
}

void unregister(bk_ctx* c) {
  if (c->pinned_data && c->host) cudaHostUnregister((void*)c->host);
  if (c->pinned_off && c->off) cudaHostUnregister((void*)c->off);
  c->pinned_data = c->pinned_off = c->registered = false;
  c->host = nullptr;
  c->off = nullptr;
  c->host_dev = nullptr;
  c->n = c->nbytes = 0;
}

}  // namespace

extern "C" {

const char* bk_strerror(int status) {
  switch (status) {
    case BK_OK: return "ok";
    case BK_E_INVAL: return "invalid argument";
    case BK_E_NOMEM: return "out of memory / window too small";
    case BK_E_CUDA: return "CUDA error";
    case BK_E_STATE: return "bad call order";
    case BK_E_RANGE: return "record exceeds chunk budget";
    case BK_E_CAPACITY: return "output capacity too small";
    case BK_E_UNSUPPORTED: return "unsupported";
    default: return "unknown status";
  }
}

const char* bk_last_error(void) { return g_last_error.c_str(); }

int bk_create(const bk_config* cfg, bk_ctx** out_ctx) {
  if (!cfg || !out_ctx) return fail(BK_E_INVAL, "NULL argument");
  if (cfg->struct_size != sizeof(bk_config)) return fail(BK_E_INVAL, "bk_config size %u != %zu", cfg->struct_size, sizeof(bk_config));
  *out_ctx = nullptr;
  bk_ctx* c = new (std::nothrow) bk_ctx();
  if (!c) return fail(BK_E_NOMEM, "host allocation");
  c->cfg = *cfg;
  if (!c->cfg.window_bytes) c->cfg.window_bytes = 2ull << 30;
  if (!c->cfg.n_slots) c->cfg.n_slots = 4;
  if (c->cfg.n_slots < 2 || c->cfg.n_slots > 64) { delete c; return fail(BK_E_INVAL, "n_slots must be in 2..64"); }
  if (c->cfg.lanes % 32) { delete c; return fail(BK_E_INVAL, "lanes must be a multiple of 32"); }
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || c->cfg.device < 0 || c->cfg.device >= ndev) {
    cudaGetLastError();
    delete c;
    return fail(BK_E_CUDA, "no CUDA device %d", cfg->device);
  }
  c->cfg.window_bytes = c->cfg.window_bytes / (c->cfg.n_slots * kAlign) * (c->cfg.n_slots * kAlign);
  auto cleanup = [&](int rc) { bk_destroy(c); return rc; };
  if (cudaSetDevice(c->cfg.device) != cudaSuccess) return cleanup(fail(BK_E_CUDA, "cudaSetDevice"));
  if (configure_compute_kernels() != cudaSuccess) return cleanup(fail(BK_E_CUDA, "cudaFuncSetAttribute"));
  if (cudaStreamCreateWithFlags(&c->s_copy, cudaStreamNonBlocking) != cudaSuccess ||
      cudaStreamCreateWithFlags(&c->s_asm, cudaStreamNonBlocking) != cudaSuccess ||
      cudaStreamCreateWithFlags(&c->s_comp, cudaStreamNonBlocking) != cudaSuccess ||
      cudaEventCreateWithFlags(&c->ev_begin, cudaEventDisableTiming) != cudaSuccess ||
      cudaEventCreateWithFlags(&c->ev_end, cudaEventDisableTiming) != cudaSuccess ||
      cudaEventCreate(&c->t_begin) != cudaSuccess || cudaEventCreate(&c->t_end) != cudaSuccess)
    return cleanup(fail(BK_E_CUDA, "stream/event creation"));
  if (cudaMalloc(&c->window, c->cfg.window_bytes) != cudaSuccess) {
    cudaGetLastError();
    return cleanup(fail(BK_E_NOMEM, "cudaMalloc window %llu B", (unsigned long long)c->cfg.window_bytes));
  }
  if (cudaMalloc(&c->d_err, 256) != cudaSuccess || cudaMalloc(&c->d_ctr, 8 * sizeof(unsigned long long)) != cudaSuccess)
    return cleanup(fail(BK_E_NOMEM, "cudaMalloc scratch"));
  c->slots.resize(c->cfg.n_slots);
  if (cudaStreamCreateWithFlags(&c->s_d2h, cudaStreamNonBlocking) != cudaSuccess) return cleanup(fail(BK_E_CUDA, "d2h stream"));
  if (configure_partition_kernels() != cudaSuccess || configure_baseline_kernels() != cudaSuccess)
    return cleanup(fail(BK_E_CUDA, "cudaFuncSetAttribute"));
  if (cudaEventCreateWithFlags(&c->ev_fork, cudaEventDisableTiming) != cudaSuccess)
    return cleanup(fail(BK_E_CUDA, "events"));
  c->ev_join.assign(3 + c->cfg.n_slots, nullptr);
  for (auto& e : c->ev_join)
    if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) return cleanup(fail(BK_E_CUDA, "events"));
  c->ev_part.assign(c->cfg.n_slots, nullptr);
  for (auto& e : c->ev_part)
    if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) return cleanup(fail(BK_E_CUDA, "events"));
  c->s_slot.assign(c->cfg.n_slots, nullptr);
  for (auto& st : c->s_slot)
    if (cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking) != cudaSuccess) return cleanup(fail(BK_E_CUDA, "slot streams"));
  for (auto& s : c->slots) {
    if (cudaEventCreateWithFlags(&s.copied, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&s.ready, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&s.freed, cudaEventDisableTiming) != cudaSuccess)
      return cleanup(fail(BK_E_CUDA, "slot events"));
  }
  c->st.struct_size = sizeof(bk_stats);
  c->st.n_slots = c->cfg.n_slots;
  c->st.slot_bytes = c->cfg.window_bytes / c->cfg.n_slots;
  *out_ctx = c;
  return BK_OK;
}

int bk_register_segments(bk_ctx* c, const void* host_ptr, uint64_t nbytes, const uint64_t* off, uint64_t n) {
  if (!c) return fail(BK_E_INVAL, "NULL ctx");
  if (!host_ptr && nbytes) return fail(BK_E_INVAL, "NULL host_ptr");
  const auto t0 = std::chrono::steady_clock::now();
  if (cudaSetDevice(c->cfg.device) != cudaSuccess) return fail(BK_E_CUDA, "cudaSetDevice");
  unregister(c);
  uint64_t maxr = 0, minr = ~0ull;
  if (off) {
    if (n && off[0] != 0) return fail(BK_E_INVAL, "record_offsets[0] != 0");
    for (uint64_t i = 0; i < n; ++i) {
      const uint64_t e = i + 1 < n ? off[i + 1] : nbytes;
      if (e < off[i] || e > nbytes) return fail(BK_E_INVAL, "record_offsets not non-decreasing / > nbytes at %llu", (unsigned long long)i);
      maxr = std::max(maxr, e - off[i]);
      minr = std::min(minr, e - off[i]);
    }
    if (!n && nbytes) return fail(BK_E_INVAL, "bytes without records");
  } else if (n == 0 && nbytes == 0) {
    maxr = minr = 0;  // empty data set
  } else {
    const uint64_t rs = c->cfg.record_size;
    if (!rs) return fail(BK_E_INVAL, "record_offsets == NULL needs cfg.record_size");
    if (nbytes % rs) return fail(BK_E_INVAL, "nbytes %% record_size != 0");
    if (n != nbytes / rs) return fail(BK_E_INVAL, "n_records != nbytes / record_size");
    maxr = minr = rs;
  }
  if (!n) minr = 0;
  c->max_rec = maxr;
  c->min_rec = n ? minr : ~0ull;
  if (nbytes) {
    if (is_pinned(host_ptr)) {
      c->pinned_data = false;
    } else {
      cudaError_t e = cudaHostRegister((void*)host_ptr, nbytes, cudaHostRegisterMapped | cudaHostRegisterPortable);
      if (e != cudaSuccess) return fail(BK_E_CUDA, "cudaHostRegister(data, %llu): %s", (unsigned long long)nbytes, cudaGetErrorString(e));
      c->pinned_data = true;
    }
    void* dptr = nullptr;
    cudaError_t e = cudaHostGetDevicePointer(&dptr, (void*)host_ptr, 0);
    if (e != cudaSuccess) {
      if (c->pinned_data) cudaHostUnregister((void*)host_ptr);
      c->pinned_data = false;
      return fail(BK_E_CUDA, "cudaHostGetDevicePointer (memory pinned without cudaHostRegisterMapped?): %s", cudaGetErrorString(e));
    }
    c->host_dev = (const uint8_t*)dptr;
  }
  if (off && n) {
    if (is_pinned(off)) {
      c->pinned_off = false;
    } else {
      cudaError_t e = cudaHostRegister((void*)off, n * 8, cudaHostRegisterMapped | cudaHostRegisterPortable);
      if (e != cudaSuccess) return fail(BK_E_CUDA, "cudaHostRegister(offsets): %s", cudaGetErrorString(e));
      c->pinned_off = true;
    }
  }
  c->host = (const uint8_t*)host_ptr;
  c->nbytes = nbytes;
  c->off = off;
  c->n = n;
  c->registered = true;
  c->plan_cache.clear();
  drop_graphs(c);
  c->st.ms_register = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  return BK_OK;
}

int bk_run(bk_ctx* c, int kernel_id, void* stream, void* out) {
  if (!c || !out) return fail(BK_E_INVAL, "NULL argument");
  if (!c->registered) return fail(BK_E_STATE, "bk_run before bk_register_segments");
  const bk_out_header* h = (const bk_out_header*)out;
  if (h->kernel_id != kernel_id) return fail(BK_E_INVAL, "out->kernel_id %d != %d", h->kernel_id, kernel_id);
  const auto t0 = std::chrono::steady_clock::now();
  int rc;
  if (c->cfg.flags & (BK_FLAG_BASELINE_DBUF | BK_FLAG_BASELINE_SBUF)) {
    rc = run_dbuf(c, kernel_id, out, stream);
    if (rc) {
      cudaDeviceSynchronize();
      cudaGetLastError();
      return rc;
    }
    c->st.kernel_launches = (uint64_t)c->n_launch;
    c->st.ms_run = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    return BK_OK;
  }
  switch (kernel_id) {
    case BK_K_WORDCOUNT:
      if (h->struct_size != sizeof(bk_out_wordcount)) return fail(BK_E_INVAL, "bk_out_wordcount size");
      rc = run_wordcount(c, (bk_out_wordcount*)out, stream);
      break;
    case BK_K_GREP:
      if (h->struct_size != sizeof(bk_out_grep)) return fail(BK_E_INVAL, "bk_out_grep size");
      rc = run_grep(c, (bk_out_grep*)out, stream);
      break;
    case BK_K_KMEANS:
      if (h->struct_size != sizeof(bk_out_kmeans)) return fail(BK_E_INVAL, "bk_out_kmeans size");
      rc = run_kmeans(c, (bk_out_kmeans*)out, stream);
      break;
    case BK_K_GROUPBY:
      if (h->struct_size != sizeof(bk_out_groupby)) return fail(BK_E_INVAL, "bk_out_groupby size");
      rc = run_groupby(c, (bk_out_groupby*)out, stream);
      break;
    case BK_K_KMER:
      if (h->struct_size != sizeof(bk_out_kmer)) return fail(BK_E_INVAL, "bk_out_kmer size");
      rc = run_kmer(c, (bk_out_kmer*)out, stream);
      break;
    case BK_K_PATTERN_STATS:
      if (h->struct_size != sizeof(bk_out_pattern)) return fail(BK_E_INVAL, "bk_out_pattern size");
      rc = run_pattern(c, (bk_out_pattern*)out, stream);
      break;
    case BK_K_LAYOUT_DUMP:
      if (h->struct_size != sizeof(bk_out_layout)) return fail(BK_E_INVAL, "bk_out_layout size");
      rc = run_layout(c, (bk_out_layout*)out, stream);
      break;
    case BK_K_PARTITION:
      if (h->struct_size != sizeof(bk_out_partition)) return fail(BK_E_INVAL, "bk_out_partition size");
      rc = run_partition(c, (bk_out_partition*)out, stream);
      break;
    default:
      return fail(BK_E_UNSUPPORTED, "unknown kernel_id %d", kernel_id);
  }
  if (rc) {
    // leave the context usable: drain whatever was queued
    cudaStreamSynchronize(c->s_copy);
    cudaStreamSynchronize(c->s_asm);
    cudaStreamSynchronize(c->s_comp);
    for (auto st : c->s_slot) cudaStreamSynchronize(st);
    cudaGetLastError();
    return rc;
  }
  c->st.kernel_launches = (uint64_t)c->n_launch;
  c->st.ms_run = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  return BK_OK;
}

int bk_get_stats(const bk_ctx* c, bk_stats* s) {
  if (!c || !s) return fail(BK_E_INVAL, "NULL argument");
  if (s->struct_size != sizeof(bk_stats)) return fail(BK_E_INVAL, "bk_stats size");
  *s = c->st;
  return BK_OK;
}

int bk_abi_sizes(uint32_t* sizes, int n) {
  const uint32_t v[10] = {sizeof(bk_config),     sizeof(bk_out_wordcount), sizeof(bk_out_grep),
                          sizeof(bk_out_kmeans), sizeof(bk_out_partition), sizeof(bk_out_groupby),
                          sizeof(bk_out_layout), sizeof(bk_stats),         sizeof(bk_out_pattern),
                          sizeof(bk_out_kmer)};
  for (int i = 0; i < n && i < 10; ++i) sizes[i] = v[i];
  return BK_ABI_VERSION;
}

int bk_destroy(bk_ctx* c) {
  if (!c) return BK_OK;
  cudaSetDevice(c->cfg.device);
  if (c->s_comp) cudaStreamSynchronize(c->s_comp);
  if (c->s_copy) cudaStreamSynchronize(c->s_copy);
  if (c->s_asm) cudaStreamSynchronize(c->s_asm);
  for (auto st : c->s_slot)
    if (st) cudaStreamSynchronize(st);
  unregister(c);
  for (auto& s : c->slots) {
    if (s.copied) cudaEventDestroy(s.copied);
    if (s.ready) cudaEventDestroy(s.ready);
    if (s.freed) cudaEventDestroy(s.freed);
  }
  for (DevBuf* b : {&c->b_table, &c->b_out1, &c->b_out2, &c->b_out3, &c->b_blk, &c->b_blk2, &c->b_agg1, &c->b_agg2,
                    &c->b_agg3, &c->b_mu})
    b->release();
  if (c->window) cudaFree(c->window);
  if (c->d_err) cudaFree(c->d_err);
  if (c->d_ctr) cudaFree(c->d_ctr);
  if (c->ev_begin) cudaEventDestroy(c->ev_begin);
  if (c->ev_end) cudaEventDestroy(c->ev_end);
  if (c->t_begin) cudaEventDestroy(c->t_begin);
  if (c->t_end) cudaEventDestroy(c->t_end);
  for (cudaEvent_t e : c->prof) cudaEventDestroy(e);
  drop_graphs(c);
  if (c->ev_fork) cudaEventDestroy(c->ev_fork);
  for (auto e : c->ev_join) cudaEventDestroy(e);
  if (c->h_mu) cudaFreeHost(c->h_mu);
  delete c->pool;
  if (c->s_d2h) {
    cudaStreamSynchronize(c->s_d2h);
    cudaStreamDestroy(c->s_d2h);
  }
  for (auto e : c->ev_part) cudaEventDestroy(e);
  for (auto& e : c->out_pinned) cudaHostUnregister(e.first);
  for (DevBuf* b : {&c->b_hist, &c->b_colpre, &c->b_totals, &c->b_base}) b->release();
  for (auto* h : c->hstage) cudaFreeHost(h);
  for (auto e : c->h_done) cudaEventDestroy(e);
  if (c->s_copy) cudaStreamDestroy(c->s_copy);
  if (c->s_asm) cudaStreamDestroy(c->s_asm);
  if (c->s_comp) cudaStreamDestroy(c->s_comp);
  for (auto st : c->s_slot)
    if (st) cudaStreamDestroy(st);
  cudaGetLastError();
  delete c;
  return BK_OK;
}

}  // extern "C"
