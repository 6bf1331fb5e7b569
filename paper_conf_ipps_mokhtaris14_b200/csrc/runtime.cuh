// runtime.cuh — internal host-side definitions of libbk's runtime (context, plan, ring slots,
// CUDA-graph cache) shared by the runtime translation units:
//   runtime_plan.cu      chunk + lane planning, slot carving (a1)
//   runtime_pipeline.cu  stages 1-3 per chunk, event ring, fork/join, stats, graphs (a2-a4, a6)
//   runtime_kernels.cu   the per-kernel drivers (a5, a7) and the experiment kernels
//   runtime_api.cu       the C ABI of include/bk.h (a0: create / register / run / destroy)
//
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
#pragma once
#include <cuda_runtime.h>
#include <nvtx3/nvToolsExt.h>   // header-only NVTX v3: ranges cost ~ns when no tool is attached

#include <algorithm>
#include <chrono>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>
#include <string>
#include <thread>
#include <utility>
#include <vector>

#include "../../include/bk.h"
#include "bk_internal.cuh"
#include "host_gather.h"
#include "trace.h"

namespace bk {
namespace rt {

// Sets the thread-local detail string of bk_last_error() and returns `code`.
int fail(int code, const char* fmt, ...);

#define BK_CUDA(expr)                                                                        \
  do {                                                                                       \
    cudaError_t e_ = (expr);                                                                 \
    if (e_ != cudaSuccess)                                                                   \
      return ::bk::rt::fail(BK_E_CUDA, "%s failed: %s (%s:%d)", #expr, cudaGetErrorString(e_), __FILE__, __LINE__); \
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
  // BK_GATHER_ADDR: explicit addresses (device staging), per-lane explicit counts and their scan;
  // bk_run_user_addr: the generator's address buffer, per-lane bases and counts
  uint64_t* exp = nullptr;
  uint32_t* ecount = nullptr;
  uint64_t* epos = nullptr;
  uint64_t* uaddr = nullptr;
  uint64_t* ubase = nullptr;
  uint32_t* ucount = nullptr;
  // descriptor sets (meta, lanes, tileK, tile_base); ZC plans keep two so that stage 1 of chunk
  // i+N can run while chunk i still computes from the other set. meta..tile_base above point at
  // the set of the chunk being issued.
  uint64_t* meta_set[2] = {nullptr, nullptr};
  LaneDesc* lanes_set[2] = {nullptr, nullptr};
  uint32_t* tileK_set[2] = {nullptr, nullptr};
  uint64_t* tile_base_set[2] = {nullptr, nullptr};
  cudaEvent_t copied = nullptr, ready = nullptr, freed = nullptr;
  cudaEvent_t zt0 = nullptr, zt1 = nullptr;   // HYBRID: device time of the slot's zero-copy gather
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
  uint32_t desc_sets = 1;              // descriptor sets per slot (2: ZC, stage 1 runs a chunk ahead)
  bool packed = false;                 // CPU chunks: host packs records' bytes, GPU interleaves (raw slot)
  uint32_t elem = 0;                   // BK_GATHER_ADDR: bytes per element address
  uint64_t exp_cap = 0;                // BK_GATHER_ADDR: bytes of one chunk's addresses (8 per element)
  bool user_addr = false;              // bk_run_user_addr: the caller's generator writes the addresses
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

}  // namespace rt
}  // namespace bk

struct bk_ctx {  // the opaque context of include/bk.h
  bk_config cfg{};
  cudaStream_t s_copy = nullptr, s_asm = nullptr, s_comp = nullptr;
  std::vector<cudaStream_t> s_slot;  // per-slot compute streams for commutative kernels
  std::vector<cudaStream_t> s_stage; // per-slot zero-copy staging streams (stages 1-3 of slot k's chunks)
  cudaEvent_t ev_begin = nullptr, ev_end = nullptr;
  cudaEvent_t t_begin = nullptr, t_end = nullptr;   // timing events on s_comp (device time of a run)
  std::vector<cudaEvent_t> prof;                   // BK_FLAG_PROFILE: per chunk x stage begin/end
  std::vector<int> prof_stage;                     // stage id of each event pair
  size_t prof_used = 0;
  size_t prof_open[8] = {};                        // event index of each stage's open pair
  uint8_t* window = nullptr;    // the whole streaming working set (cfg.window_bytes)
  std::vector<bk::rt::Slot> slots;
  // registration
  const uint8_t* host = nullptr;
  uint64_t nbytes = 0;
  const uint64_t* off = nullptr;
  uint64_t n = 0;
  bool pinned_data = false, pinned_off = false, registered = false;
  bool registered_ro = false;          // the data set was registered cudaHostRegisterReadOnly
  const uint8_t* host_dev = nullptr;   // device alias of the mapped data set
  const uint64_t* off_dev = nullptr;   // device alias of the mapped offsets (nullptr: not mapped)
  uint64_t max_rec = 0, min_rec = 0;
  // device scratch / resident buffers
  int* d_err = nullptr;
  unsigned long long* d_ctr = nullptr;  // [0] staged sum, [1] wc used, [2] wc n_out, [3] grep running, [4] kmeans chk
  // pinned mirror of d_ctr[0..7] and d_err (at [8]), copied by the run's tail before its one sync
  unsigned long long* h_ctr = nullptr;
  bk::rt::DevBuf b_table, b_out1, b_out2, b_out3, b_blk, b_blk2, b_blk3, b_agg1, b_agg2, b_agg3, b_mu;
  // CPU assembly (BK_GATHER_CPU / HYBRID): thread pool + pinned host staging ring
  bk::HostPool* pool = nullptr;
  std::vector<uint8_t*> hstage;
  std::vector<cudaEvent_t> h_done;
  std::vector<bool> h_used;
  uint64_t hstage_cap = 0;
  uint64_t h_next = 0;
  std::vector<uint64_t> scratch_first, scratch_tiles;
  // partition: D2H stream, per-slot "kernels done" events, resident totals, pinned output cache
  cudaStream_t s_d2h = nullptr;
  std::vector<cudaEvent_t> ev_part;
  bk::rt::DevBuf b_hist, b_colpre, b_totals, b_base;
  bk::rt::DevBuf b_h1, b_h2;                 // word-count key hashes (multi-GPU merge keys)
  bk::rt::DevBuf b_units;                    // BK_GATHER_FUSED unit plan (record bounds, byte bounds)
  bk::rt::DevBuf b_flags;                    //   ring ready / done flags
  bk::rt::DevBuf b_batch;                    //   DMA feed: batch plan (byte / record bounds, unit -> batch)
  bk::rt::DevBuf b_kbin;                     // k-mers: coarse bins of phase A
  std::string batch_key;
  uint64_t n_batches = 0;
  std::vector<uint64_t> h_bby, h_brec;
  cudaEvent_t ev_fused = nullptr;
  std::string units_key;                     //   which plan b_units holds
  uint64_t n_units = 0;
  unsigned long long* d_fprof = nullptr;     //   in-kernel wait / compute counters
  // BK_GATHER_ADDR: per slot, pinned + mapped host memory the GPU writes the address information to
  // (the paper's CPU-side addrBuf), and the host's view of the chunk's tiles
  std::vector<bk::AddrDesc*> a_desc_h, a_desc_d;
  std::vector<uint64_t*> a_exp_h, a_exp_d, a_tot_h, a_tot_d;
  uint64_t a_exp_cap = 0, a_L = 0;
  std::vector<cudaEvent_t> a_ready;          // per slot: stage 1 (addresses) of its chunk finished
  size_t addr_next = 0;                      // next chunk whose stage 1 is not yet issued
  std::vector<uint64_t> a_epos, a_tbase;
  std::vector<bk::trace::Rec> trace_recs;    // BK_FLAG_TRACE: this run's CUPTI records
  bool tracing = false;
  double hy_t_zc_ms = 0, hy_t_cpu_ms = 0;    // HYBRID: measured ms per zero-copy / host-packed chunk
  void* wc_clean_ptr = nullptr;              // word count: b_table is all zero in its first
  uint64_t wc_clean_slots = 0;               //   wc_clean_slots entries (drained by the last run)
  bk_addr_fn a_gen = nullptr;                // bk_run_user_addr generator + its argument
  void* a_gen_user = nullptr;
  bk::rt::DevBuf b_mown, b_mcnt, b_mctr;     // bk_merge_counts scratch (never captured in a graph)
  std::vector<std::pair<void*, uint64_t>> out_pinned;      // caller output arrays pinned across runs (opt-in)
  std::vector<std::pair<void*, uint64_t>> out_pinned_run;  // caller output arrays pinned for this run only
  int n_launch = 0;
  bk_stats st{};
  std::vector<std::pair<std::string, bk::rt::Plan>> plan_cache;
  std::vector<bk::rt::GraphEntry> graphs;
  cudaEvent_t ev_fork = nullptr;
  std::vector<cudaEvent_t> ev_join;
  float* h_mu = nullptr;   // pinned copy of the k-means centroids (graph memcpy source)
  uint64_t test_rng = 0x9E3779B97F4A7C15ull;   // BK_FLAG_TEST_DELAYS
};


namespace bk {
namespace rt {

// ---- planning (runtime_plan.cu)
bool is_pinned(const void* p);
uint64_t rec_start(const bk_ctx* c, uint64_t r);
int make_chunks(const bk_ctx* c, Plan& p);
int plan_run(bk_ctx* c, const Access& a, uint32_t lane_target, Plan& p, uint32_t out_per_chunk = 0,
             int auto_mode = BK_GATHER_AUTO, bool user_addr = false);
void carve(bk_ctx* c, const Plan& p);
Chunk chunk_of(const bk_ctx* c, const Plan& p, size_t i);
Access whole_access();
Access field_access(uint32_t off, uint32_t len);
int parse_access(const bk_ctx* c, uint32_t n_ext, const uint32_t* eo, const uint32_t* el, Access& a);

// ---- pipeline (runtime_pipeline.cu)
enum { kStH2D = 0, kStAddrgen = 1, kStGather = 2, kStCompute = 3, kStRelayout = 4, kStD2H = 5, kNStages = 6 };
int prof_mark(bk_ctx* c, int stage, cudaStream_t s, bool begin);
#define BK_PROF(stage, stream, begin) do { int r_ = prof_mark(c, stage, stream, begin); if (r_) return r_; } while (0)
uint64_t test_rand(bk_ctx* c);
#define BK_DELAY(stream)                                                                      \
  do {                                                                                        \
    if (c->cfg.flags & BK_FLAG_TEST_DELAYS) launch_spin((long long)(::bk::rt::test_rand(c) % 200000), stream); \
  } while (0)
int ensure_host_side(bk_ctx* c, const Plan& p);
int ensure_addr_side(bk_ctx* c, const Plan& p);
int stage_chunk_addr(bk_ctx* c, const Plan& p, size_t i, Slot& s);
void release_addr_side(bk_ctx* c);
int stage_chunk_cpu(bk_ctx* c, const Plan& p, size_t i, Slot& s);
int stage_chunk(bk_ctx* c, const Plan& p, size_t i, Slot& s);
void note_plan(bk_ctx* c, const Plan& p);
int check_err(bk_ctx* c);
int begin_run(bk_ctx* c, void* stream);
int end_run(bk_ctx* c, void* stream);
int device_begin(bk_ctx* c);
int device_end(bk_ctx* c);
void host_reset(bk_ctx* c);
int prof_reserve(bk_ctx* c, size_t pairs);
int refork(bk_ctx* c);   // compute streams wait for everything enqueued on s_comp so far
int end_host(bk_ctx* c, void* stream);
int trace_begin(bk_ctx* c);
void drop_graphs(bk_ctx* c);
bool graphable(const Plan& p);
// Stage 4 stages tiles through TMA bulk copies unless zero-copy gathers run alongside (ZC, HYBRID):
// those keep the SMs' sysmem path busy and the bulk copies were measured to stall behind them.
inline bool stage_tma(const Plan& p) { return p.mode == BK_GATHER_DENSE || p.mode == BK_GATHER_CPU; }
int ensure_out_pinned(bk_ctx* c, void* ptr, uint64_t bytes);
void* out_kernel_ptr(bk_ctx* c, void* ptr, uint64_t bytes);
void release_run_outputs(bk_ctx* c);
void release_kept_outputs(bk_ctx* c);
void unregister(bk_ctx* c);

// NVTX ranges (SURVEY §5 tracing): bk_run / registration, and per chunk its stage issue ("chunk i
// zc|cpu|dense") and compute enqueue, so `ncu --nvtx --nvtx-include "bk_run.grep/"` or a timeline
// tool can select one workload's kernels. They mark host issue time; GPU time is in bk_stats.
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  template <class... A>
  NvtxRange(const char* fmt, A... a) {
    char b[96];
    snprintf(b, sizeof b, fmt, a...);
    nvtxRangePushA(b);
  }
  ~NvtxRange() { nvtxRangePop(); }
  NvtxRange(const NvtxRange&) = delete;
  NvtxRange& operator=(const NvtxRange&) = delete;
};

template <class Compute>
int pipeline(bk_ctx* c, const Plan& p, bool concurrent, Compute&& compute) {
  const size_t C = p.bounds.size() - 1;
  c->st.n_chunks = C;
  note_plan(c, p);
  // HYBRID adaptive split: zero-copy chunks in flight while the host packs one chunk. Starts at one
  // (16 host threads pack a chunk faster than the link gathers one zero-copy: profiles/r01_hybrid_sweep.md)
  // and follows the measured ratio (host time per packed chunk) / (time per zero-copy chunk), so a rank
  // with few host cores (8 ranks on one host) lets the GPU gather more and never waits on slow packers.
  std::vector<Slot*> zc_inflight;
  size_t zc_depth = 1;
  double& t_zc_ms = c->hy_t_zc_ms;    // running estimates, kept across runs of one registration
  double& t_cpu_ms = c->hy_t_cpu_ms;
  if (p.mode == BK_GATHER_CPU || p.mode == BK_GATHER_HYBRID || p.mode == BK_GATHER_ADDR) {
    int rc = ensure_host_side(c, p);
    if (!rc && p.mode == BK_GATHER_ADDR) rc = ensure_addr_side(c, p);
    if (rc) return rc;
  }
  c->addr_next = 0;
  if (int rf = refork(c)) return rf;   // the driver's setup on s_comp happens-before every chunk's compute
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
      // adaptive split (default): the GPU zero-copy gathers run asynchronously; keep zc_depth in
      // flight and let the host pool assemble the next chunk while they are busy
      while (!zc_inflight.empty() && cudaEventQuery(zc_inflight.front()->ready) == cudaSuccess) {
        float ms = 0;   // the gather's own device time (timing events around it)
        if (cudaEventElapsedTime(&ms, zc_inflight.front()->zt0, zc_inflight.front()->zt1) == cudaSuccess && ms > 0)
          t_zc_ms = t_zc_ms > 0 ? 0.5 * (t_zc_ms + ms) : ms;
        zc_inflight.erase(zc_inflight.begin());
      }
      cudaGetLastError();
      if (t_zc_ms > 0 && t_cpu_ms > 0)
        zc_depth = (size_t)std::max<long>(1, std::min<long>((long)c->cfg.n_slots - 1, std::lround(t_cpu_ms / t_zc_ms)));
      cpu = zc_inflight.size() >= zc_depth;
      // a packed chunk earns one chunk per t_cpu but idles the link for t_cpu - (N-1) t_zc once the
      // zero-copy chunks in flight drain: pack only while that pays (t_cpu < N t_zc); else ZC only
      if (t_zc_ms > 0 && t_cpu_ms > (double)c->cfg.n_slots * t_zc_ms) cpu = false;
    }
    int rc;
    {
      NvtxRange r("chunk %zu %s", i, p.mode == BK_GATHER_ADDR ? "addr" : cpu ? "cpu" : p.zero_copy ? "zc" : "dense");
      const double packed0 = c->st.ms_cpu_gather;   // host time of the packing itself (no waits)
      rc = p.mode == BK_GATHER_ADDR ? stage_chunk_addr(c, p, i, s) : cpu ? stage_chunk_cpu(c, p, i, s)
                                                                          : stage_chunk(c, p, i, s);
      if (cpu && p.mode == BK_GATHER_HYBRID && !rc) {
        const double ms = c->st.ms_cpu_gather - packed0;
        t_cpu_ms = t_cpu_ms > 0 ? 0.5 * (t_cpu_ms + ms) : ms;
      }
    }
    if (rc) return rc;
    if (p.mode == BK_GATHER_HYBRID && !cpu) zc_inflight.push_back(&s);
    BK_CUDA(cudaStreamWaitEvent(cs, s.ready, 0));
    BK_DELAY(cs);
    BK_PROF(kStCompute, cs, true);
    cudaStream_t rel = cs;   // stream whose completion frees the slot (partition: its D2H)
    {
      NvtxRange r("compute %zu", i);
      rc = compute(chunk_of(c, p, i), s, cs, rel);
    }
    if (rc) return rc;
    BK_PROF(kStCompute, cs, false);
    BK_CUDA(cudaEventRecord(s.freed, rel));
  }
  if (concurrent)  // join: finalize on s_comp after every slot's last compute
    for (auto& s : c->slots)
      if (s.used) BK_CUDA(cudaStreamWaitEvent(c->s_comp, s.freed, 0));
  return BK_OK;
}


// Every device address a captured graph may bake in besides those the per-kernel key already names
// (the window's carving is a function of the plan, which is in the key): the resident DevBufs can be
// reallocated by a later run with larger parameters, so their current addresses are part of the key
// and a graph whose buffers moved is never replayed (it would touch freed memory).
std::string resident_key(const bk_ctx* c);
std::string mem_key(const void* p);   // address + CUDA allocation id of a caller buffer a graph bakes in
constexpr size_t kMaxGraphs = 16;   // cached graphs per context (oldest dropped first)

template <class Enqueue>
int run_device(bk_ctx* c, void* stream, const std::string& key_in, bool graphable, size_t n_chunks, Enqueue&& enqueue) {
  BK_CUDA(cudaSetDevice(c->cfg.device));
  const std::string key = key_in + "|" + resident_key(c);
  host_reset(c);
  if (int rt = trace_begin(c)) return rt;
  BK_CUDA(cudaEventRecord(c->ev_begin, (cudaStream_t)stream));
  BK_CUDA(cudaStreamWaitEvent(c->s_comp, c->ev_begin, 0));
  BK_CUDA(cudaEventRecord(c->t_begin, c->s_comp));
  int rc;
  // per-stage profiling events must be real stream events (timestamps), so BK_FLAG_PROFILE issues eagerly
  // outputs registered for this run only are unregistered at its end: a graph of their copies could
  // never be replayed (mem_key differs next run), so such runs issue eagerly instead of capturing
  if (!graphable || !c->out_pinned_run.empty() || (c->cfg.flags & (BK_FLAG_NO_GRAPH | BK_FLAG_PROFILE))) {
    if ((rc = device_begin(c)) || (rc = enqueue()) || (rc = device_end(c))) return rc;
    c->st.graph_issue = 0;
    return end_host(c, stream);
  }
  GraphEntry* ge = nullptr;
  for (auto& g : c->graphs)
    if (g.key == key) ge = &g;
  const bool replay = ge != nullptr;
  if (ge) {
    const double reg = c->st.ms_register;
    c->st = ge->st;
    c->st.ms_register = reg;
    c->n_launch = ge->n_launch;
    c->prof_used = ge->prof_used;
    for (size_t i = 0; i < ge->prof_stage.size(); ++i) c->prof_stage[i] = ge->prof_stage[i];
  } else {
    if ((rc = prof_reserve(c, 5 * n_chunks + 8))) return rc;
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
    if (c->graphs.size() >= kMaxGraphs) {
      if (c->graphs.front().exec) cudaGraphExecDestroy(c->graphs.front().exec);
      c->graphs.erase(c->graphs.begin());
    }
    c->graphs.push_back(std::move(g));
    ge = &c->graphs.back();
  }
  c->st.graph_issue = replay ? 2 : 1;
  BK_CUDA(cudaGraphLaunch(ge->exec, c->s_comp));
  return end_host(c, stream);
}


// ---- kernel drivers (runtime_kernels.cu)
int run_wordcount(bk_ctx* c, bk_out_wordcount* o, void* stream);
int run_grep(bk_ctx* c, bk_out_grep* o, void* stream);
int run_groupby(bk_ctx* c, bk_out_groupby* o, void* stream);
int run_kmeans(bk_ctx* c, bk_out_kmeans* o, void* stream);
int run_kmer(bk_ctx* c, bk_out_kmer* o, void* stream);
int run_partition(bk_ctx* c, bk_out_partition* o, void* stream);
int run_dbuf(bk_ctx* c, int kid, void* out, void* stream);
int run_pattern(bk_ctx* c, bk_out_pattern* o, void* stream);
int run_layout(bk_ctx* c, bk_out_layout* o, void* stream);
int run_user(bk_ctx* c, const bk_access* a, bk_chunk_fn fn, void* user, void* stream);
int run_user_addr(bk_ctx* c, const bk_access* a, bk_addr_fn gen, void* gen_user, bk_chunk_fn fn, void* user,
                  void* stream);

}  // namespace rt
}  // namespace bk
