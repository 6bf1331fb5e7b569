// runtime_kernels.cu — per-kernel drivers: plan, resident buffers, the enqueue lambda for the
// pipeline, result copies into the caller's out struct; the double-buffering
// baseline and the experiment kernels (layout dump, pattern statistics).
#include "runtime.cuh"

#include <cuda.h>   // CUstream / CUdeviceptr types of the stream memory operations

namespace bk {
namespace rt {

// ------------------------------------------------------------------ kernels

// Where k_wc_compact stores the distinct words: straight into the caller's arrays when kernels can
// reach all of them (device memory, or pinned / kept-pinned host memory through its mapped alias:
// the PCIe stores replace a copy after the run), else into HBM staging copied by wordcount_results.
struct WcOut {
  uint64_t* off;
  uint32_t* len;
  uint64_t* cnt;
  uint64_t* h1;
  uint64_t* h2;
  bool direct;
  std::string key() const {
    return direct ? "/d" + mem_key(off) + "." + mem_key(len) + "." + mem_key(cnt) + "." + mem_key(h1) + "." + mem_key(h2)
                  : "/s" + std::to_string(h1 != nullptr);
  }
};

static WcOut wordcount_out(bk_ctx* c, bk_out_wordcount* o, uint64_t ocap) {
  WcOut w{};
  w.off = (uint64_t*)out_kernel_ptr(c, o->word_off, ocap * 8);
  w.len = w.off ? (uint32_t*)out_kernel_ptr(c, o->word_len, ocap * 4) : nullptr;
  w.cnt = w.len ? (uint64_t*)out_kernel_ptr(c, o->word_count, ocap * 8) : nullptr;
  w.h1 = o->word_h1 && w.cnt ? (uint64_t*)out_kernel_ptr(c, o->word_h1, ocap * 8) : nullptr;
  w.h2 = o->word_h2 && w.cnt ? (uint64_t*)out_kernel_ptr(c, o->word_h2, ocap * 8) : nullptr;
  w.direct = w.cnt && (!o->word_h1 || w.h1) && (!o->word_h2 || w.h2);
  if (!w.direct) {
    w.off = (uint64_t*)c->b_out1.p;
    w.len = (uint32_t*)c->b_out2.p;
    w.cnt = (uint64_t*)c->b_out3.p;
    w.h1 = o->word_h1 ? (uint64_t*)c->b_h1.p : nullptr;
    w.h2 = o->word_h2 ? (uint64_t*)c->b_h2.p : nullptr;
  }
  return w;
}

// distinct words + totals of the finished run -> the caller's (host or device) arrays
static int wordcount_results(bk_ctx* c, bk_out_wordcount* o, uint64_t slots, bool direct) {
  const unsigned long long nw = c->h_ctr[2];
  o->n_words = nw;
  if (nw > o->cap) return fail(BK_E_CAPACITY, "%llu distinct words > cap %llu", nw, (unsigned long long)o->cap);
  if (nw * 2 > slots) return fail(BK_E_CAPACITY, "table load %llu/%llu too high; raise table_slots", nw,
                                  (unsigned long long)slots);
  if (nw && !direct) {   // host or device result arrays (unified addressing)
    BK_CUDA(cudaMemcpy(o->word_off, c->b_out1.p, nw * 8, cudaMemcpyDefault));
    BK_CUDA(cudaMemcpy(o->word_len, c->b_out2.p, nw * 4, cudaMemcpyDefault));
    BK_CUDA(cudaMemcpy(o->word_count, c->b_out3.p, nw * 8, cudaMemcpyDefault));
    if (o->word_h1) BK_CUDA(cudaMemcpy(o->word_h1, c->b_h1.p, nw * 8, cudaMemcpyDefault));
    if (o->word_h2) BK_CUDA(cudaMemcpy(o->word_h2, c->b_h2.p, nw * 8, cudaMemcpyDefault));
  }
  o->total_words = c->h_ctr[6];
  c->st.bytes_d2h = nw * (20 + (o->word_h1 ? 8 : 0) + (o->word_h2 ? 8 : 0));
  return BK_OK;
}

// The word-count table between runs: k_wc_compact zeroes every slot it drains, so after a completed
// run the table's first `slots` entries are zero and the next run skips the 32-MB memset. The memset
// runs (eagerly, ahead of the run's graph on the compute stream) when the table is new or grown, was
// used by another kernel (k-mers, the baselines), or the last run did not complete.
static int wc_table_begin(bk_ctx* c, uint64_t slots) {
  const bool clean = c->wc_clean_ptr == c->b_table.p && c->wc_clean_slots >= slots;
  c->wc_clean_ptr = nullptr;   // dirty until this run's compaction has completed
  if (!clean) BK_CUDA(cudaMemsetAsync(c->b_table.p, 0, slots * sizeof(WcEntry), c->s_comp));
  return BK_OK;
}
static void wc_table_end(bk_ctx* c, uint64_t slots) {
  c->wc_clean_ptr = c->b_table.p;
  c->wc_clean_slots = slots;
}

// BK_GATHER_FUSED unit plan: greedy whole records, each unit <= UB bytes and <= UR records (A3 with a
// second cap: shared-memory slots hold the unit's offsets too). 0 on success, BK_E_RANGE when a
// record exceeds UB (the caller falls back to the event pipeline).
static int fused_units(bk_ctx* c, uint32_t UB, uint32_t UR, std::vector<uint64_t>& ub, std::vector<uint64_t>& uby) {
  ub.assign(1, 0);
  uby.assign(1, 0);
  uint64_t lo = 0;
  while (lo < c->n) {
    uint64_t hi = lo;
    const uint64_t b0 = rec_start(c, lo);
    if (!c->off) {
      const uint64_t k = std::min<uint64_t>(UB / c->cfg.record_size, UR);
      if (k == 0) return BK_E_RANGE;
      hi = std::min<uint64_t>(c->n, lo + k);
    } else {
      const uint64_t lim = b0 + UB;
      const uint64_t rmax = std::min<uint64_t>(c->n, lo + UR);
      while (hi < rmax && rec_start(c, hi + 1) <= lim) ++hi;
      if (hi == lo) return BK_E_RANGE;
    }
    ub.push_back(hi);
    uby.push_back(rec_start(c, hi));
    lo = hi;
  }
  return BK_OK;
}

// Stream memory operations (driver API through the runtime's entry-point query, no -lcuda): the
// copy stream writes a flag after each batch's DMA and waits for the consumers' release flag — the
// paper's "DMA a flag right after the data" and its buffer-reuse distance.
namespace {
using PfnStreamValue64 = CUresult (*)(CUstream, CUdeviceptr, cuuint64_t, unsigned int);
struct MemOps {
  bool tried = false;
  PfnStreamValue64 write = nullptr, wait = nullptr;
};
MemOps& memops() {
  static MemOps m;
  if (!m.tried) {
    m.tried = true;
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuStreamWriteValue64", &f, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      m.write = reinterpret_cast<PfnStreamValue64>(f);
    if (cudaGetDriverEntryPoint("cuStreamWaitValue64", &f, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      m.wait = reinterpret_cast<PfnStreamValue64>(f);
    cudaGetLastError();
  }
  return m;
}
}  // namespace

// Word count as one persistent launch (BK_GATHER_FUSED, kernels_compute.cu k_wc_fused): loader
// CTAs stream units into an HBM ring carved from the window, consumer CTAs count. Returns
// BK_E_RANGE (nothing enqueued) when the window cannot hold a ring of >= 2 units or a record does
// not fit a unit: the caller then runs the event pipeline.
static int run_wordcount_fused(bk_ctx* c, bk_out_wordcount* o, void* stream, uint64_t slots, uint64_t ocap,
                               const WcOut& wo) {
  (void)o;
  const int grid = wc_fused_grid();
  if (grid < 2) return BK_E_RANGE;
  uint32_t n_load = (uint32_t)std::max(1, grid / 4);   // sweeps r02e/r02h: 24-49 of 148 loaders saturate the link
  if (const char* e = getenv("BK_FUSED_LOADERS")) n_load = (uint32_t)std::max(1, std::min(grid - 1, atoi(e)));
  // units as large as 16 KiB allow while the ring keeps >= 2 slots per CTA; >= 2 KiB units and
  // >= 2 slots in any case (R x slot <= window_bytes)
  uint64_t UB = c->cfg.window_bytes / (2ull * grid);
  UB = UB > 64 ? (UB - 64) * 2 / 3 : 0;
  uint64_t ub_max = 16384;
  if (const char* e = getenv("BK_FUSED_UNIT")) ub_max = std::max<uint64_t>(2048, std::min<uint64_t>(65536, atoll(e)));
  UB = std::max<uint64_t>(2048, std::min<uint64_t>(UB, ub_max)) / 16 * 16;
  if (c->cfg.chunk_bytes) UB = std::min<uint64_t>(UB, c->cfg.chunk_bytes / 16 * 16);   // explicit unit cap
  if (UB < 16) return BK_E_RANGE;
  const uint32_t UR = (uint32_t)std::max<uint64_t>(UB / 16, 16);
  if (c->cfg.flags & BK_FLAG_TEST_DELAYS) return BK_E_RANGE;   // delay injection targets the event pipeline
  const uint64_t slot_bytes = wc_fused_slot_bytes((uint32_t)UB, UR);
  const uint64_t R = std::min<uint64_t>(c->cfg.window_bytes / slot_bytes, 1u << 20);
  if (R < 2) return BK_E_RANGE;
  const std::string ukey = std::to_string(UB) + "/" + std::to_string(UR);
  if (c->units_key != ukey) {
    std::vector<uint64_t> ub, uby;
    if (fused_units(c, (uint32_t)UB, UR, ub, uby)) return BK_E_RANGE;
    c->n_units = ub.size() - 1;
    BK_CUDA(c->b_units.ensure(2 * ub.size() * 8));
    BK_CUDA(cudaMemcpy(c->b_units.p, ub.data(), ub.size() * 8, cudaMemcpyHostToDevice));
    BK_CUDA(cudaMemcpy((uint64_t*)c->b_units.p + ub.size(), uby.data(), uby.size() * 8, cudaMemcpyHostToDevice));
    c->units_key = ukey;
  }
  if (!c->d_fprof) BK_CUDA(cudaMalloc(&c->d_fprof, 8 * 8));
  // feed: "zc" (default): loader CTAs stream units with zero-copy loads; "dma" (BK_FUSED_FEED=dma):
  // the copy engine fills K batch slots, each followed by a stream-ordered flag, every CTA consumes.
  // Measured on the C1 config (profiles/r02_wc_fused.md): zc 1.74 ms/step, dma 1.88 (K=2) - 2.15 (K=4):
  // the batch-granular release leaves the copy engine waiting at every batch boundary.
  const char* fe = getenv("BK_FUSED_FEED");
  const bool dma = fe && strcmp(fe, "dma") == 0 && memops().write && memops().wait;
  uint32_t K = 3;
  if (const char* e = getenv("BK_FUSED_BATCHES")) K = (uint32_t)std::max(2, std::min(8, atoi(e)));
  const uint64_t bslot = c->cfg.window_bytes / K / 256 * 256;
  const uint64_t btext = (bslot * 7 / 8 - 64) / 16 * 16;
  const uint64_t brecs = (bslot - btext - 64) / 8;
  FusedDma fd{};
  if (dma) {
    if (btext < UB || brecs < UR) return BK_E_RANGE;
    const std::string bkey = ukey + "/" + std::to_string(K) + "/" + std::to_string(bslot);
    if (c->batch_key != bkey) {
      const uint64_t* hub = nullptr;
      std::vector<uint64_t> ubh(c->n_units + 1), ubyh(c->n_units + 1);
      BK_CUDA(cudaMemcpy(ubh.data(), c->b_units.p, ubh.size() * 8, cudaMemcpyDeviceToHost));
      BK_CUDA(cudaMemcpy(ubyh.data(), (uint64_t*)c->b_units.p + ubh.size(), ubh.size() * 8, cudaMemcpyDeviceToHost));
      (void)hub;
      std::vector<uint32_t> ubatch(c->n_units), bunits;
      std::vector<uint64_t> bby{0}, brec{0};
      uint64_t u0 = 0;
      while (u0 < c->n_units) {   // greedy: consecutive units while the batch's bytes and records fit a slot
        uint64_t u1 = u0 + 1;
        while (u1 < c->n_units && ubyh[u1 + 1] - ubyh[u0] + 16 <= btext && ubh[u1 + 1] - ubh[u0] <= brecs) ++u1;
        for (uint64_t u = u0; u < u1; ++u) ubatch[u] = (uint32_t)bunits.size();
        bunits.push_back((uint32_t)(u1 - u0));
        bby.push_back(ubyh[u1]);
        brec.push_back(ubh[u1]);
        u0 = u1;
      }
      c->n_batches = bunits.size();
      c->h_bby = bby;
      c->h_brec = brec;
      const size_t NB = c->n_batches;
      BK_CUDA(c->b_batch.ensure(c->n_units * 4 + NB * 4 + 2 * (NB + 1) * 8 + 64));
      uint8_t* q = (uint8_t*)c->b_batch.p;
      BK_CUDA(cudaMemcpy(q, bby.data(), (NB + 1) * 8, cudaMemcpyHostToDevice));
      BK_CUDA(cudaMemcpy(q + (NB + 1) * 8, brec.data(), (NB + 1) * 8, cudaMemcpyHostToDevice));
      BK_CUDA(cudaMemcpy(q + 2 * (NB + 1) * 8, ubatch.data(), c->n_units * 4, cudaMemcpyHostToDevice));
      BK_CUDA(cudaMemcpy(q + 2 * (NB + 1) * 8 + c->n_units * 4, bunits.data(), NB * 4, cudaMemcpyHostToDevice));
      c->batch_key = bkey;
    }
    uint8_t* q = (uint8_t*)c->b_batch.p;
    const size_t NB = c->n_batches;
    fd.bby = (const uint64_t*)q;
    fd.brec = (const uint64_t*)(q + (NB + 1) * 8);
    fd.ubatch = (const uint32_t*)(q + 2 * (NB + 1) * 8);
    fd.bunits = (const uint32_t*)(q + 2 * (NB + 1) * 8 + c->n_units * 4);
    fd.K = K;
    fd.bslot_bytes = bslot;
    fd.btext = btext;
  }
  BK_CUDA(c->b_flags.ensure(2 * std::max<uint64_t>(R, K) * 8 + K * 4 + 64));
  const uint64_t U = c->n_units;
  const uint64_t* ubd = (const uint64_t*)c->b_units.p;
  const uint64_t NF = dma ? K : R;   // flags per direction
  unsigned long long* ready = (unsigned long long*)c->b_flags.p;
  fd.bcnt = (unsigned int*)(ready + 2 * NF);
  const bool prof = (c->cfg.flags & BK_FLAG_PROFILE) != 0;
  WcEntry* table = (WcEntry*)c->b_table.p;
  // captured once per (table, units, ring, loaders) and replayed: two memsets, the cooperative
  // persistent kernel, the compaction
  const std::string key = "wcfused/" + std::to_string(slots) + "/" + std::to_string(ocap) + "/" + ukey + "/" +
                          std::to_string(R) + "/" + std::to_string(n_load) + wo.key();
  // the DMA feed issues eagerly (stream memory operations are not graph-captured here)
  if (int r0 = wc_table_begin(c, slots)) return r0;
  int rc = run_device(c, stream, key + (dma ? "/dma" : "/zc"), !dma, 1, [&]() -> int {
    BK_CUDA(cudaMemsetAsync(ready, 0, 2 * NF * 8 + K * 4, c->s_comp));
    if (prof) BK_CUDA(cudaMemsetAsync(c->d_fprof, 0, 8 * 8, c->s_comp));
    if (dma) {   // the copy stream starts after the flags are cleared
      BK_CUDA(cudaEventRecord(c->ev_fused, c->s_comp));
      BK_CUDA(cudaStreamWaitEvent(c->s_copy, c->ev_fused, 0));
    }
    BK_PROF(kStGather, c->s_comp, true);
    BK_CUDA(launch_wc_fused(c->host_dev, c->nbytes, c->off ? c->off_dev : nullptr, c->off ? 0 : c->cfg.record_size,
                            ubd, ubd + U + 1, (uint32_t)U, (uint32_t)UB, UR, grid, dma ? 0 : n_load, c->window,
                            (uint32_t)R, ready, ready + NF, table, slots - 1, c->d_ctr + 1, c->d_err,
                            prof ? c->d_fprof : nullptr, dma ? &fd : nullptr, c->s_comp));
    BK_PROF(kStGather, c->s_comp, false);
    if (dma) {   // per batch: [wait for the slot's release] -> DMA text + offsets -> flag (stream order)
      const MemOps& mo = memops();
      for (size_t b = 0; b < c->n_batches; ++b) {
        const uint64_t sl = b % K;
        uint8_t* slot = c->window + sl * bslot;
        if (b >= K && mo.wait((CUstream)c->s_copy, (CUdeviceptr)(ready + NF + sl), b - K + 1, CU_STREAM_WAIT_VALUE_GEQ))
          return fail(BK_E_CUDA, "cuStreamWaitValue64");
        const uint64_t b0 = c->h_bby[b], b1 = c->h_bby[b + 1];
        BK_CUDA(cudaMemcpyAsync(slot + (((uintptr_t)(c->host_dev + b0)) & 15), c->host + b0, b1 - b0,
                                cudaMemcpyHostToDevice, c->s_copy));
        if (c->off)
          BK_CUDA(cudaMemcpyAsync(slot + btext + 64, c->off + c->h_brec[b], (c->h_brec[b + 1] - c->h_brec[b]) * 8,
                                  cudaMemcpyHostToDevice, c->s_copy));
        if (mo.write((CUstream)c->s_copy, (CUdeviceptr)(ready + sl), b + 1, CU_STREAM_WRITE_VALUE_DEFAULT))
          return fail(BK_E_CUDA, "cuStreamWriteValue64");
      }
    }
    launch_wc_compact(table, slots, c->d_ctr + 2, c->d_ctr + 6, wo.off, wo.len, wo.cnt, wo.h1, wo.h2, ocap, c->s_comp);
    c->n_launch += 2;
    return (int)BK_OK;
  });
  if (rc) return rc;
  wc_table_end(c, slots);
  c->st.gather_mode = BK_GATHER_FUSED;
  c->st.chunk_budget = UB;
  c->st.n_chunks = U;
  c->st.lanes = wc_fused_threads();
  c->st.bytes_accessed = c->nbytes;
  c->st.bytes_h2d = c->nbytes;
  c->st.bytes_meta = c->off ? c->n * 8 : 0;
  c->st.n_chunks_zc = U;
  c->st.bytes_zc = c->nbytes;
  c->st.records_zc = c->n;
  c->st.n_units = U;
  c->st.unit_bytes = (uint32_t)UB;
  c->st.fused_grid = (uint32_t)grid;
  c->st.fused_loaders = dma ? 0 : n_load;
  c->st.fused_ring_slots = dma ? K : (uint32_t)R;
  c->st.fused_wait_frac = c->st.fused_compute_frac = c->st.fused_loader_wait_frac = 0;
  if (prof) {
    unsigned long long fp[5] = {0, 0, 0, 0, 0};
    BK_CUDA(cudaMemcpy(fp, c->d_fprof, sizeof fp, cudaMemcpyDeviceToHost));
    if (fp[2]) {
      c->st.fused_wait_frac = (double)fp[0] / (double)fp[2];   // consumers
      c->st.fused_compute_frac = (double)fp[1] / (double)fp[2];
    }
    if (fp[3] + fp[4]) c->st.fused_loader_wait_frac = (double)fp[3] / (double)(fp[3] + fp[4]);
    // the one kernel is stages 1-4: its interval is the transfer interval; the consumers' compute
    // share of it overlaps the loaders' transfers of later units
    c->st.ms_compute_busy = c->st.ms_zc * c->st.fused_compute_frac;
    c->st.ms_compute = c->st.ms_compute_busy;
    c->st.ms_overlap = c->st.ms_compute_busy;
  }
  return BK_OK;
}

int run_wordcount(bk_ctx* c, bk_out_wordcount* o, void* stream) {
  uint64_t slots = o->table_slots ? o->table_slots : (1ull << 20);
  if (slots & (slots - 1)) return fail(BK_E_INVAL, "table_slots must be a power of two");
  const uint64_t ocap0 = std::min<uint64_t>(o->cap, slots);
  // FUSED: when asked for, or AUTO's pick unless the caller fixed the chunking (chunk_bytes / lanes)
  const bool fused = c->cfg.gather_mode == BK_GATHER_FUSED ||
                     (c->cfg.gather_mode == BK_GATHER_AUTO && !c->cfg.chunk_bytes && !c->cfg.lanes);
  if (fused && c->n) {
    BK_CUDA(c->b_table.ensure(slots * sizeof(WcEntry)));
    BK_CUDA(c->b_out1.ensure(std::max<uint64_t>(ocap0, 1) * 8));
    BK_CUDA(c->b_out2.ensure(std::max<uint64_t>(ocap0, 1) * 4));
    BK_CUDA(c->b_out3.ensure(std::max<uint64_t>(ocap0, 1) * 8));
    BK_CUDA(c->b_h1.ensure(std::max<uint64_t>(ocap0, 1) * 8));
    BK_CUDA(c->b_h2.ensure(std::max<uint64_t>(ocap0, 1) * 8));
    const WcOut wo = wordcount_out(c, o, ocap0);
    const int frc = run_wordcount_fused(c, o, stream, slots, ocap0, wo);
    if (frc == BK_OK) return wordcount_results(c, o, slots, wo.direct);
    if (frc != BK_E_RANGE) return frc;
  }
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
  BK_CUDA(c->b_h1.ensure(std::max<uint64_t>(ocap, 1) * 8));
  BK_CUDA(c->b_h2.ensure(std::max<uint64_t>(ocap, 1) * 8));
  WcEntry* table = (WcEntry*)c->b_table.p;
  const WcOut wo = wordcount_out(c, o, ocap);
  const std::string key = "wc/" + std::to_string(slots) + "/" + std::to_string(ocap) + "/" + p.key + wo.key();
  if ((rc = wc_table_begin(c, slots))) return rc;
  rc = run_device(c, stream, key, graphable(p), p.bounds.size() - 1, [&]() -> int {
    int r = pipeline(c, p, true, [&](const Chunk& ch, Slot& s, cudaStream_t cs, cudaStream_t&) {
      launch_wc(ch, s.stage, s.lanes, s.tile_base, s.meta, c->off ? 0 : c->cfg.record_size, table, slots - 1,
                c->d_ctr + 1, c->d_err, cs);
      c->n_launch += 1;
      return BK_OK;
    });
    if (r) return r;
    launch_wc_compact(table, slots, c->d_ctr + 2, c->d_ctr + 6, wo.off, wo.len, wo.cnt, wo.h1, wo.h2, ocap, c->s_comp);
    c->n_launch += 1;
    return (int)BK_OK;
  });
  if (rc) return rc;
  wc_table_end(c, slots);
  return wordcount_results(c, o, slots, wo.direct);
}

int run_grep(bk_ctx* c, bk_out_grep* o, void* stream) {
  if (o->pattern_len > 32) return fail(BK_E_INVAL, "pattern longer than 32 bytes");
  if (o->pattern_len && !o->pattern) return fail(BK_E_INVAL, "NULL pattern");
  if (c->min_rec < 48) return fail(BK_E_INVAL, "grep needs records of >= 48 bytes (key at +16..+48)");
  Plan p;
  int rc = plan_run(c, field_access(16, 32), 256, p);
  if (rc) return rc;
  carve(c, p);
  const uint32_t ntl = std::max<uint32_t>(p.L / 32, 1);   // tiles per chunk (L % 32 == 0)
  const uint64_t cap = std::min<uint64_t>(o->cap, c->n);
  const size_t C = p.bounds.size() - 1;
  const uint32_t N = c->cfg.n_slots;
  BK_CUDA(c->b_out1.ensure(std::max<uint64_t>(cap, 1) * 8));   // matches in chunk order
  BK_CUDA(c->b_out2.ensure(std::max<uint64_t>(cap, 1) * 8));   // match pool (runs in completion order)
  BK_CUDA(c->b_out3.ensure(std::max<size_t>(C, 1) * 16));       // per chunk {pool offset, count}
  BK_CUDA(c->b_blk.ensure((uint64_t)ntl * 4 * N));              // per slot: tile match counts
  BK_CUDA(c->b_blk2.ensure((uint64_t)ntl * 8 * N));             // per slot: tile output bases
  BK_CUDA(c->b_blk3.ensure((uint64_t)ntl * 32 * 4 * N));        // per slot: lane match masks
  const int dev_sms = device_sms();
  const int grid = dev_sms * 2;   // 2 x 8-warp blocks per SM stream the tiles (64 KB smem each)
  GrepParams gp{};
  if (o->pattern_len) memcpy(gp.pat, o->pattern, o->pattern_len);
  gp.plen = o->pattern_len;
  gp.first_index = o->first_index;
  gp.cap = cap;
  std::string key = "grep/" + std::to_string(gp.plen) + "/" + std::to_string(gp.first_index) + "/" +
                    std::to_string(gp.cap) + "/" + p.key + "/";
  for (uint32_t i = 0; i < gp.plen; ++i) key += std::to_string(gp.pat[i]) + ",";
  rc = run_device(c, stream, key, graphable(p), p.bounds.size() - 1, [&]() -> int {
    size_t ci = 0;
    int r = pipeline(c, p, true, [&](const Chunk& ch, Slot& s, cudaStream_t cs, cudaStream_t&) {
      const size_t k = ci % N;   // slot of this chunk: its block counts/bases are private to it
      launch_grep(ch, s.stage, s.lanes, s.tile_base, gp, (uint32_t*)c->b_blk.p + k * ntl,
                  (uint32_t*)c->b_blk3.p + k * ntl * 32, c->d_ctr + 3, (unsigned long long*)c->b_blk2.p + k * ntl,
                  (unsigned long long*)c->b_out3.p + 2 * ci, (uint64_t*)c->b_out2.p, c->d_err, grid, stage_tma(p), cs);
      ++ci;
      c->n_launch += 3;
      return BK_OK;
    });
    if (r) return r;
    launch_grep_order((const unsigned long long*)c->b_out3.p, (uint32_t)C, (const uint64_t*)c->b_out2.p,
                      (uint64_t*)c->b_out1.p, cap, c->s_comp);
    c->n_launch += 1;
    return (int)BK_OK;
  });
  if (rc) return rc;
  unsigned long long m = 0;
  m = c->h_ctr[3];
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
  const int dev_sms = device_sms();
  int per_sm = 1;
  const bool tma = stage_tma(p);
  per_sm = std::max<int>(1, (int)((220 * 1024) / std::max<size_t>(groupby_smem(G, tma), 1)));
  per_sm = std::min(per_sm, 3);
  const int grid = std::max(1, std::min<int>((p.L + 255) / 256, dev_sms * per_sm));
  rc = run_device(c, stream, "groupby/" + std::to_string(G) + "/" + p.key, graphable(p), p.bounds.size() - 1,
                  [&]() -> int {
    BK_CUDA(cudaMemsetAsync(c->b_agg1.p, 0, (uint64_t)G * 8, c->s_comp));
    BK_CUDA(cudaMemsetAsync(c->b_agg2.p, 0, (uint64_t)G * 8, c->s_comp));
    BK_CUDA(cudaMemsetAsync(c->b_agg3.p, 0, (uint64_t)G * 8, c->s_comp));
    return pipeline(c, p, true, [&](const Chunk& ch, Slot& s, cudaStream_t cs, cudaStream_t&) {
      launch_groupby(ch, s.stage, s.lanes, s.tile_base, G, (unsigned long long*)c->b_agg1.p,
                     (unsigned long long*)c->b_agg2.p, (double*)c->b_agg3.p, c->d_err, grid, tma, cs);
      c->n_launch += 1;
      return BK_OK;
    });
  });
  if (rc) return rc;
  BK_CUDA(cudaMemcpy(o->count, c->b_agg1.p, (uint64_t)G * 8, cudaMemcpyDefault));
  BK_CUDA(cudaMemcpy(o->qty, c->b_agg2.p, (uint64_t)G * 8, cudaMemcpyDefault));
  BK_CUDA(cudaMemcpy(o->amount, c->b_agg3.p, (uint64_t)G * 8, cudaMemcpyDefault));
  c->st.bytes_d2h = (uint64_t)G * 24;
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
  const int dev_sms = device_sms();
  if (!c->h_mu) BK_CUDA(cudaHostAlloc((void**)&c->h_mu, 256 * 64, cudaHostAllocPortable));
  memcpy(c->h_mu, o->centroids, (size_t)K * 64);   // the graph copies from this pinned buffer
  const bool tma = stage_tma(p);   // TMA: one 16-warp block per SM; plain loads: two
  const int grid = std::max(1, std::min<int>((p.L + 255) / 256, dev_sms * (tma ? 1 : 2)));
  const std::string key = "kmeans/" + std::to_string(K) + "/" + std::to_string(o->first_index) + "/" +
                          mem_key(o->cid) + "/" + p.key;
  rc = run_device(c, stream, key, graphable(p), p.bounds.size() - 1, [&]() -> int {
    BK_CUDA(cudaMemcpyAsync(c->b_mu.p, c->h_mu, (uint64_t)K * 64, cudaMemcpyHostToDevice, c->s_comp));
    BK_CUDA(cudaMemsetAsync(c->b_agg1.p, 0, (uint64_t)K * 8, c->s_comp));
    BK_CUDA(cudaMemsetAsync(c->b_agg3.p, 0, (uint64_t)K * 128, c->s_comp));
    size_t ci = 0;
    return pipeline(c, p, true, [&](const Chunk& ch, Slot& s, cudaStream_t cs, cudaStream_t& rel) -> int {
      launch_kmeans(ch, s.stage, s.lanes, s.tile_base, (const float*)c->b_mu.p, K, o->first_index,
                    (unsigned long long*)c->b_agg1.p, (double*)c->b_agg3.p, c->d_ctr + 4,
                    o->cid ? (int32_t*)s.out : nullptr, grid, tma, cs);
      c->n_launch += 1;
      if (o->cid && ch.hi > ch.lo) {  // write-back of this chunk's cids, full duplex with the H2D stream
        cudaEvent_t e = c->ev_part[ci++ % c->ev_part.size()];
        BK_CUDA(cudaEventRecord(e, cs));
        BK_CUDA(cudaStreamWaitEvent(c->s_d2h, e, 0));
        BK_PROF(kStD2H, c->s_d2h, true);
        BK_CUDA(cudaMemcpyAsync(o->cid + ch.lo, s.out, (ch.hi - ch.lo) * 4, cudaMemcpyDeviceToHost, c->s_d2h));
        BK_PROF(kStD2H, c->s_d2h, false);
        c->st.bytes_d2h += (ch.hi - ch.lo) * 4;
        rel = c->s_d2h;
      }
      return (int)BK_OK;
    });
  });
  if (rc) return rc;
  BK_CUDA(cudaMemcpy(o->count, c->b_agg1.p, (uint64_t)K * 8, cudaMemcpyDefault));
  BK_CUDA(cudaMemcpy(o->sum, c->b_agg3.p, (uint64_t)K * 128, cudaMemcpyDefault));
  unsigned long long chk = 0;
  chk = c->h_ctr[4];
  o->chk = chk;
  c->st.bytes_d2h += (uint64_t)K * 136;
  return BK_OK;
}

// f4: k-mer counting (FIELD access to the sequence; the table is resident, outside the window).
// Two-phase (kernels_kmer.cu): per chunk every k-mer key is appended to its table region's bucket,
// and flushes count whole buckets into their regions in shared memory.
int run_kmer(bk_ctx* c, bk_out_kmer* o, void* stream) {
  c->wc_clean_ptr = nullptr;   // the table buffer holds k-mer regions now
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
  // the final flush stores the distinct k-mers straight into the caller's arrays when kernels can
  // reach them (device memory, or pinned host memory through its mapped alias: the PCIe stores then
  // overlap the flush instead of following it as a copy); else into HBM, copied after the run
  uint64_t* dk = (uint64_t*)out_kernel_ptr(c, o->kmer, ocap * 8);
  uint64_t* dc = dk ? (uint64_t*)out_kernel_ptr(c, o->count, ocap * 8) : nullptr;
  const bool direct = dk && dc;
  if (!direct) {
    BK_CUDA(c->b_out1.ensure(std::max<uint64_t>(ocap, 1) * 8));
    BK_CUDA(c->b_out3.ensure(std::max<uint64_t>(ocap, 1) * 8));
    dk = (uint64_t*)c->b_out1.p;
    dc = (uint64_t*)c->b_out3.p;
  }
  KmerEntry* table = (KmerEntry*)c->b_table.p;
  // regions of <= 8192 slots (96 KiB of shared memory in the flush: 2 CTAs per SM). Phase A bins keys into 2^cb <= 256
  // coarse bins (one global atomic per block step and bin); the flush splits them into the regions'
  // buckets (cb < rb), then counts each bucket in its region. Buckets are sized for the run's k-mer
  // windows (an upper bound: every window of every record valid) within 16 GiB each, else flushed every
  // F chunks; a full bucket falls back to direct inserts
  const uint64_t S = std::min<uint64_t>(slots, 8192);
  uint32_t rb = 0;
  while ((S << rb) < slots) ++rb;
  const uint64_t R = 1ull << rb;
  const uint32_t cb = std::min<uint32_t>(rb, 8);
  const uint64_t NB = 1ull << cb;
  const bool two = cb < rb;
  const uint64_t wpr = o->seq_len >= o->k ? o->seq_len - o->k + 1 : 0;   // windows per record (bound)
  const uint64_t bound = c->n * wpr;
  const uint64_t fbudget = std::min<uint64_t>(16ull << 30, (uint64_t)(bound * 1.15) * 8 + R * 8192 + 8);
  const uint32_t fcap = (uint32_t)std::min<uint64_t>(fbudget / 8 / R, 0xffffffffull);
  const uint64_t cbudget = two ? std::min<uint64_t>(16ull << 30, (uint64_t)(bound * 1.1) * 8 + NB * 65536 + 8) : 0;
  const uint32_t ccap = two ? (uint32_t)std::min<uint64_t>(cbudget / 8 / NB, 0xffffffffull) : 0;
  uint64_t per_chunk = 0;
  for (size_t i = 0; i + 1 < p.bounds.size(); ++i) per_chunk = std::max<uint64_t>(per_chunk, (p.bounds[i + 1] - p.bounds[i]) * wpr);
  const uint64_t cap_keys = two ? std::min<uint64_t>((uint64_t)ccap * NB, (uint64_t)fcap * R) : (uint64_t)fcap * R;
  // per_chunk is an upper bound (every window valid), so F chunks always fit the buckets on average;
  // a region's share above its bucket's 15% + 8192-key margin goes to the region directly (exact)
  uint64_t F = per_chunk ? std::max<uint64_t>(1, cap_keys / per_chunk) : 1;
  if (getenv("BK_KMER_F")) F = std::max<uint64_t>(1, std::min<uint64_t>(F, (uint64_t)atoll(getenv("BK_KMER_F"))));
  // split each chunk's coarse bins right after binning it (chunks then run in order on one stream), so
  // the split overlaps the transfer of later chunks instead of lengthening the final flush (measured:
  // 60.3 vs 65.9 ms per 4-GiB step, profiles/r02_kmer.md); BK_KMER_SPLIT_EACH=0 splits once per flush
  const char* se = getenv("BK_KMER_SPLIT_EACH");
  const bool split_each = two && !(se && atoi(se) == 0);
  BK_CUDA(c->b_blk.ensure((uint64_t)fcap * R * 8));
  if (two) BK_CUDA(c->b_kbin.ensure((uint64_t)ccap * NB * 8));
  BK_CUDA(c->b_blk2.ensure(R * 5 + NB * 8 + 64));
  unsigned long long* bbuf = (unsigned long long*)c->b_blk.p;
  unsigned int* bcur = (unsigned int*)c->b_blk2.p;
  unsigned char* dirty = (unsigned char*)(bcur + R);
  unsigned int* ccur = (unsigned int*)((uint8_t*)c->b_blk2.p + (R * 5 + 15) / 16 * 16);
  unsigned int* cdone = ccur + NB;
  unsigned long long* cbuf = two ? (unsigned long long*)c->b_kbin.p : bbuf;
  const std::string key = "kmer/" + std::to_string(o->k) + "/" + std::to_string(slots) + "/" + std::to_string(ocap) +
                          "/" + std::to_string(F) + "/" + std::to_string(split_each) + "/" + mem_key(dk) + "/" + mem_key(dc) + "/" + p.key;
  rc = run_device(c, stream, key, graphable(p), p.bounds.size() - 1, [&]() -> int {
    BK_CUDA(cudaMemsetAsync(c->b_table.p, 0, slots * sizeof(KmerEntry), c->s_comp));
    BK_CUDA(cudaMemsetAsync(c->b_blk2.p, 0, R * 5 + NB * 8 + 64, c->s_comp));   // cursors, dirty flags
    auto split = [&](cudaStream_t st) {
      launch_kmer_split(cbuf, ccur, ccap, cdone, rb, cb, bbuf, bcur, fcap, table, S, dirty, c->d_err, st);
      c->n_launch += 1;
    };
    auto flush = [&](int final_flush, cudaStream_t st) {
      if (two && !split_each) split(st);
      launch_kmer_flush(table, rb, S, bbuf, bcur, fcap, dirty, final_flush, dk, dc, ocap, c->d_ctr + 2, c->d_err, st);
      c->n_launch += 1;
    };
    size_t ci = 0;
    // appends commute: chunks bin concurrently unless a mid-run flush must see all of them
    const bool one_flush = F + 1 >= p.bounds.size() && !split_each;
    int r = pipeline(c, p, one_flush, [&](const Chunk& ch, Slot& s, cudaStream_t cs, cudaStream_t&) {
      launch_kmer_bin(ch, s.stage, s.lanes, s.tile_base, o->k, o->seq_len / 16, table, rb, cb, S, cbuf,
                      two ? ccur : bcur, two ? ccap : fcap, dirty, c->d_ctr + 5, c->d_err, cs);
      c->n_launch += 1;
      if (split_each) split(cs);
      if (++ci % F == 0 && ci + 1 < p.bounds.size()) flush(0, cs);   // buckets near full: count them now
      return BK_OK;
    });
    if (r) return r;
    flush(1, c->s_comp);   // final: emits the distinct k-mers
    return (int)BK_OK;
  });
  if (rc) return rc;
  unsigned long long nk = 0, tot = 0;
  nk = c->h_ctr[2];
  tot = c->h_ctr[5];
  o->n_kmers = nk;
  o->total = tot;
  if (nk > o->cap) return fail(BK_E_CAPACITY, "%llu distinct k-mers > cap %llu", nk, (unsigned long long)o->cap);
  if (nk * 10 > slots * 7) return fail(BK_E_CAPACITY, "k-mer table load %llu/%llu too high; raise table_slots", nk,
                                       (unsigned long long)slots);
  if (nk && !direct) {
    // the result arrays are large (16 B per distinct k-mer): pin them so the copy runs at DMA speed
    if ((rc = ensure_out_pinned(c, o->kmer, nk * 8)) || (rc = ensure_out_pinned(c, o->count, nk * 8))) return rc;
    BK_CUDA(cudaMemcpy(o->kmer, c->b_out1.p, nk * 8, cudaMemcpyDefault));
    BK_CUDA(cudaMemcpy(o->count, c->b_out3.p, nk * 8, cudaMemcpyDefault));
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
  const std::string key = "part/" + std::to_string(B) + "/" + mem_key(o->out_records) + "/" + p.key;
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
      if (bytes) {
        BK_PROF(kStD2H, c->s_d2h, true);
        BK_CUDA(cudaMemcpyAsync((uint8_t*)o->out_records + ch.lo * 16, s.out, bytes, cudaMemcpyDeviceToHost, c->s_d2h));
        BK_PROF(kStD2H, c->s_d2h, false);
      }
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
  c->wc_clean_ptr = nullptr;   // the baselines use the table buffer with their own memset
  if (kid != BK_K_GREP && kid != BK_K_GROUPBY && kid != BK_K_KMEANS && kid != BK_K_WORDCOUNT)
    return fail(BK_E_UNSUPPORTED, "dbuf baseline: word count / grep / group-by / k-means only");
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
  bk_out_kmeans* ok = (bk_out_kmeans*)out;
  bk_out_wordcount* ow = (bk_out_wordcount*)out;
  const uint32_t nb = dbuf_blocks();
  uint64_t wc_slots = 0, wc_ocap = 0;
  if (kid == BK_K_WORDCOUNT) {
    wc_slots = ow->table_slots ? ow->table_slots : (1ull << 20);
    if (wc_slots & (wc_slots - 1)) return fail(BK_E_INVAL, "table_slots must be a power of two");
    wc_ocap = std::min<uint64_t>(ow->cap, wc_slots);
    BK_CUDA(c->b_table.ensure(wc_slots * sizeof(WcEntry)));
    BK_CUDA(c->b_out1.ensure(std::max<uint64_t>(wc_ocap, 1) * 8));
    BK_CUDA(c->b_out2.ensure(std::max<uint64_t>(wc_ocap, 1) * 4));
    BK_CUDA(c->b_out3.ensure(std::max<uint64_t>(wc_ocap, 1) * 8));
    BK_CUDA(c->b_h1.ensure(std::max<uint64_t>(wc_ocap, 1) * 8));
    BK_CUDA(c->b_h2.ensure(std::max<uint64_t>(wc_ocap, 1) * 8));
  } else if (kid == BK_K_KMEANS) {
    if (ok->K == 0 || ok->K > 256 || !ok->centroids) return fail(BK_E_INVAL, "K must be in 1..256 with centroids");
    if (ok->cid) return fail(BK_E_UNSUPPORTED, "dbuf baseline: no k-means cid write-back");
    if (c->off || c->cfg.record_size < 64) return fail(BK_E_INVAL, "k-means needs fixed records >= 64 B");
    BK_CUDA(c->b_mu.ensure((uint64_t)ok->K * 64));
    BK_CUDA(c->b_agg1.ensure((uint64_t)ok->K * 8));
    BK_CUDA(c->b_agg3.ensure((uint64_t)ok->K * 16 * 8));
    BK_CUDA(cudaMemcpy(c->b_mu.p, ok->centroids, (uint64_t)ok->K * 64, cudaMemcpyHostToDevice));
  } else if (kid == BK_K_GREP) {
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
  if (kid == BK_K_WORDCOUNT) {
    BK_CUDA(cudaMemsetAsync(c->b_table.p, 0, wc_slots * sizeof(WcEntry), c->s_comp));
    BK_CUDA(cudaEventRecord(c->ev_begin, c->s_comp));
    BK_CUDA(cudaStreamWaitEvent(c->s_copy, c->ev_begin, 0));
    BK_CUDA(cudaStreamWaitEvent(c->s_asm, c->ev_begin, 0));
  }
  if (kid == BK_K_GROUPBY || kid == BK_K_KMEANS) {
    const uint64_t n1 = kid == BK_K_GROUPBY ? (uint64_t)ob->G * 8 : (uint64_t)ok->K * 8;
    const uint64_t n3 = kid == BK_K_GROUPBY ? (uint64_t)ob->G * 8 : (uint64_t)ok->K * 128;
    BK_CUDA(cudaMemsetAsync(c->b_agg1.p, 0, n1, c->s_comp));
    if (kid == BK_K_GROUPBY) BK_CUDA(cudaMemsetAsync(c->b_agg2.p, 0, (uint64_t)ob->G * 8, c->s_comp));
    BK_CUDA(cudaMemsetAsync(c->b_agg3.p, 0, n3, c->s_comp));
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
    } else if (kid == BK_K_WORDCOUNT) {
      launch_dbuf_wc(buf[b] + raw_off, c->off ? meta[b] : nullptr, lo, hi, base, end, c->cfg.record_size,
                     (WcEntry*)c->b_table.p, wc_slots - 1, c->d_ctr + 1, c->d_err, st);
      c->n_launch += 1;
    } else if (kid == BK_K_KMEANS) {
      launch_dbuf_kmeans(buf[b] + raw_off, lo, hi, base, c->cfg.record_size, (const float*)c->b_mu.p, ok->K,
                         ok->first_index, (unsigned long long*)c->b_agg1.p, (double*)c->b_agg3.p, c->d_ctr + 4, st);
      c->n_launch += 1;
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
  if (kid == BK_K_WORDCOUNT) {
    launch_wc_compact((WcEntry*)c->b_table.p, wc_slots, c->d_ctr + 2, c->d_ctr + 6, (uint64_t*)c->b_out1.p,
                      (uint32_t*)c->b_out2.p, (uint64_t*)c->b_out3.p, (uint64_t*)c->b_h1.p, (uint64_t*)c->b_h2.p,
                      wc_ocap, c->s_comp);
    c->n_launch += 1;
  }
  if ((rc = end_run(c, stream))) return rc;
  if (kid == BK_K_GREP) {
    unsigned long long m = 0;
    m = c->h_ctr[3];
    og->n_match = m;
    if (m > og->cap) return fail(BK_E_CAPACITY, "%llu matches > cap %llu", m, (unsigned long long)og->cap);
    if (m) BK_CUDA(cudaMemcpy(og->idx, c->b_out1.p, m * 8, cudaMemcpyDeviceToHost));
  } else if (kid == BK_K_WORDCOUNT) {
    const unsigned long long nw = c->h_ctr[2];
    ow->n_words = nw;
    if (nw > ow->cap) return fail(BK_E_CAPACITY, "%llu distinct words > cap %llu", nw, (unsigned long long)ow->cap);
    if (nw * 2 > wc_slots)
      return fail(BK_E_CAPACITY, "table load %llu/%llu too high; raise table_slots", nw, (unsigned long long)wc_slots);
    if (nw) {
      BK_CUDA(cudaMemcpy(ow->word_off, c->b_out1.p, nw * 8, cudaMemcpyDefault));
      BK_CUDA(cudaMemcpy(ow->word_len, c->b_out2.p, nw * 4, cudaMemcpyDefault));
      BK_CUDA(cudaMemcpy(ow->word_count, c->b_out3.p, nw * 8, cudaMemcpyDefault));
      if (ow->word_h1) BK_CUDA(cudaMemcpy(ow->word_h1, c->b_h1.p, nw * 8, cudaMemcpyDefault));
      if (ow->word_h2) BK_CUDA(cudaMemcpy(ow->word_h2, c->b_h2.p, nw * 8, cudaMemcpyDefault));
    }
    ow->total_words = c->h_ctr[6];
  } else if (kid == BK_K_KMEANS) {
    BK_CUDA(cudaMemcpy(ok->count, c->b_agg1.p, (uint64_t)ok->K * 8, cudaMemcpyDefault));
    BK_CUDA(cudaMemcpy(ok->sum, c->b_agg3.p, (uint64_t)ok->K * 128, cudaMemcpyDefault));
    ok->chk = c->h_ctr[4];
  } else {
    BK_CUDA(cudaMemcpy(ob->count, c->b_agg1.p, (uint64_t)ob->G * 8, cudaMemcpyDefault));
    BK_CUDA(cudaMemcpy(ob->qty, c->b_agg2.p, (uint64_t)ob->G * 8, cudaMemcpyDefault));
    BK_CUDA(cudaMemcpy(ob->amount, c->b_agg3.p, (uint64_t)ob->G * 8, cudaMemcpyDefault));
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

// bk_run_user: stages 1-3 under the caller's access spec, stage 4 enqueued by the caller per chunk.
// Always eager (no graph capture): the callback must run on every bk_run_user call.
int run_user(bk_ctx* c, const bk_access* ua, bk_chunk_fn fn, void* user, void* stream) {
  if (ua->n_ext > 8) return fail(BK_E_INVAL, "at most 8 extents");
  Access a;
  int rc = parse_access(c, ua->n_ext, ua->ext_off, ua->ext_len, a);
  if (rc) return rc;
  Plan p;
  if ((rc = plan_run(c, a, ua->lane_bytes ? ua->lane_bytes : 256, p))) return rc;
  carve(c, p);
  static_assert(sizeof(bk_lane) == sizeof(LaneDesc), "bk_lane mirrors LaneDesc");
  const size_t C = p.bounds.size() - 1;
  return run_device(c, stream, "user", false, C, [&]() -> int {
    size_t ci = 0;
    return pipeline(c, p, true, [&](const Chunk& ch, Slot& s, cudaStream_t cs, cudaStream_t&) -> int {
      bk_chunk_view v{};
      v.struct_size = sizeof(bk_chunk_view);
      v.lanes = ch.L;
      v.chunk_index = ci++;
      v.n_chunks = C;
      v.first_record = ch.lo;
      v.n_records = ch.hi - ch.lo;
      v.stage = s.stage;
      v.lane_desc = reinterpret_cast<const bk_lane*>(s.lanes);
      v.tile_base = s.tile_base;
      v.offsets = (a.whole && c->off) ? s.meta : nullptr;
      v.end_offset = ch.end_byte;
      const int r = fn(&v, (void*)cs, user);
      if (r) return fail(BK_E_INVAL, "user chunk function returned %d for chunk %llu", r,
                         (unsigned long long)v.chunk_index);
      return (int)BK_OK;
    });
  });
}

// bk_run_user_addr: the caller's generator is stage 1's address slice (address mode), stage 4 its
// chunk callback. Always eager.
int run_user_addr(bk_ctx* c, const bk_access* ua, bk_addr_fn gen, void* gen_user, bk_chunk_fn fn, void* user,
                  void* stream) {
  if (ua->n_ext > 8) return fail(BK_E_INVAL, "at most 8 extents");
  Access a;
  int rc = parse_access(c, ua->n_ext, ua->ext_off, ua->ext_len, a);
  if (rc) return rc;
  Plan p;
  if ((rc = plan_run(c, a, ua->lane_bytes ? ua->lane_bytes : 256, p, 0, BK_GATHER_AUTO, true))) return rc;
  carve(c, p);
  c->a_gen = gen;
  c->a_gen_user = gen_user;
  const size_t C = p.bounds.size() - 1;
  return run_device(c, stream, "useraddr", false, C, [&]() -> int {
    size_t ci = 0;
    return pipeline(c, p, true, [&](const Chunk& ch, Slot& s, cudaStream_t cs, cudaStream_t&) -> int {
      bk_chunk_view v{};
      v.struct_size = sizeof(bk_chunk_view);
      v.lanes = ch.L;
      v.chunk_index = ci++;
      v.n_chunks = C;
      v.first_record = ch.lo;
      v.n_records = ch.hi - ch.lo;
      v.stage = s.stage;
      v.lane_desc = reinterpret_cast<const bk_lane*>(s.lanes);
      v.tile_base = s.tile_base;
      v.offsets = c->off ? s.meta : nullptr;
      v.end_offset = ch.end_byte;
      const int r = fn(&v, (void*)cs, user);
      if (r) return fail(BK_E_INVAL, "user chunk function returned %d for chunk %llu", r,
                         (unsigned long long)v.chunk_index);
      return (int)BK_OK;
    });
  });
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
  note_plan(c, p);
  Slot& s = c->slots[p.mode == BK_GATHER_ADDR ? o->chunk % c->cfg.n_slots : 0];
  if (p.mode == BK_GATHER_ADDR) {   // stage 1 of exactly this chunk (and the look-ahead one) in its slot
    if ((rc = ensure_host_side(c, p)) || (rc = ensure_addr_side(c, p))) return rc;
    c->addr_next = o->chunk;
    if ((rc = stage_chunk_addr(c, p, o->chunk, s))) return rc;
    BK_CUDA(cudaStreamSynchronize(c->s_asm));   // the look-ahead chunk's stage 1 too
  } else if (p.mode == BK_GATHER_CPU || p.mode == BK_GATHER_HYBRID) {
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


}  // namespace rt
}  // namespace bk
