// runtime_pipeline.cu — stages 1-3 of a chunk (ZC / DENSE on the GPU, CPU assembly on the host pool),
// profiling and delay-injection hooks, fork/join of the context's streams, stage statistics and
// the CUDA-graph cache.
#include <cuda.h>   // CU_POINTER_ATTRIBUTE_BUFFER_ID (driver entry point, no -lcuda)

#include "runtime.cuh"

namespace bk {
namespace rt {

int prof_mark(bk_ctx* c, int stage, cudaStream_t s, bool begin) {
  if (!(c->cfg.flags & BK_FLAG_PROFILE)) return BK_OK;
  if (begin) {
    // a pair is claimed at its begin mark and closed through prof_open[stage], so intervals of
    // different stages may nest (the write-back D2H is issued inside the compute enqueue)
    if (c->prof_used + 2 > c->prof.size()) {
      for (int k = 0; k < 64; ++k) {
        cudaEvent_t e;
        BK_CUDA(cudaEventCreate(&e));
        c->prof.push_back(e);
        if (c->prof.size() % 2 == 0) c->prof_stage.push_back(0);
      }
    }
    c->prof_open[stage] = c->prof_used;
    c->prof_stage[c->prof_used / 2] = stage;
    BK_CUDA(cudaEventRecord(c->prof[c->prof_used], s));
    c->prof_used += 2;
  } else {
    BK_CUDA(cudaEventRecord(c->prof[c->prof_open[stage] + 1], s));
  }
  return BK_OK;
}

uint64_t test_rand(bk_ctx* c) {
  c->test_rng = c->test_rng * 6364136223846793005ull + 1442695040888963407ull;
  return c->test_rng >> 33;
}

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

// Packed CPU chunk: the host pool copies each record's accessed bytes in record order (stage 2,
// gather half), one DMA moves exactly those bytes (stage 3), and the GPU interleaves them into warp
// tiles HBM -> HBM (stage 2, layout half): the packed chunk is a run of fixed E-byte records read
// whole, so stage 1 and the whole-record gather produce the same lanes and tiles as the field plan.
static int stage_chunk_packed(bk_ctx* c, const Plan& p, size_t i, Slot& s, const Chunk& ch, const Access& a,
                              const HostData& d, size_t hs, std::chrono::steady_clock::time_point t0) {
  (void)i;
  const uint64_t size = host_pack_chunk(*c->pool, d, a, ch, c->hstage[hs], p.raw_cap);
  c->st.ms_cpu_gather += std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  if (size == UINT64_MAX) return fail(BK_E_RANGE, "host-packed chunk exceeds its slot (internal bound violated)");
  if (s.used) BK_CUDA(cudaStreamWaitEvent(c->s_copy, s.freed, 0));
  BK_DELAY(c->s_copy);
  BK_PROF(kStH2D, c->s_copy, true);
  if (size) BK_CUDA(cudaMemcpyAsync(s.raw, c->hstage[hs], size, cudaMemcpyHostToDevice, c->s_copy));
  BK_CUDA(cudaEventRecord(c->h_done[hs], c->s_copy));
  c->h_used[hs] = true;
  BK_PROF(kStH2D, c->s_copy, false);
  Chunk pc = ch;              // the packed chunk: records [lo, hi) of E bytes at raw + (r - lo) * E
  pc.base_byte = ch.lo * a.E;
  pc.end_byte = ch.hi * a.E;
  pc.guard_lo = 0;
  pc.guard_hi = p.raw_cap;
  Access pa = whole_access();
  pa.rec_size = a.E;
  BK_PROF(kStAddrgen, c->s_copy, true);
  launch_addrgen(pc, pa, s.meta, s.lanes, s.tileK, s.tile_base, p.stage_cap, c->d_err, c->d_ctr + 0, c->s_copy);
  BK_PROF(kStAddrgen, c->s_copy, false);
  BK_PROF(kStRelayout, c->s_copy, true);
  launch_gather(pc, pa, s.raw, s.meta, s.lanes, s.tile_base, s.stage, p.stage_cap, 0, c->s_copy);
  BK_PROF(kStRelayout, c->s_copy, false);
  c->n_launch += 3;
  c->st.bytes_h2d += size;
  c->st.bytes_accessed += ch.accessed;
  c->st.n_chunks_cpu += 1;
  BK_CUDA(cudaEventRecord(s.ready, c->s_copy));
  s.used = true;
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
  if (p.packed) return stage_chunk_packed(c, p, i, s, ch, a, d, hs, t0);
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

// ---- BK_GATHER_ADDR: the paper's address-mode stages 1-3 ---------------------------------------
// per slot: pinned, mapped host buffers for the lane descriptors, the explicit-address count and the
// explicit addresses (the GPU writes them, the host reads them after the slot's a_ready event)
void release_addr_side(bk_ctx* c) {
  for (auto* v : {&c->a_exp_h, &c->a_tot_h})
    for (auto* h : *v) cudaFreeHost(h);
  for (auto* h : c->a_desc_h) cudaFreeHost(h);
  c->a_desc_h.clear();
  c->a_desc_d.clear();
  c->a_exp_h.clear();
  c->a_exp_d.clear();
  c->a_tot_h.clear();
  c->a_tot_d.clear();
  for (auto e : c->a_ready) cudaEventDestroy(e);
  c->a_ready.clear();
  c->a_exp_cap = c->a_L = 0;
}

int ensure_addr_side(bk_ctx* c, const Plan& p) {
  const size_t N = c->cfg.n_slots;
  if (c->a_desc_h.size() == N && c->a_L >= p.L && c->a_exp_cap >= p.exp_cap) return BK_OK;
  release_addr_side(c);
  const unsigned fl = cudaHostAllocMapped | cudaHostAllocPortable;
  c->a_desc_h.assign(N, nullptr);
  c->a_desc_d.assign(N, nullptr);
  c->a_exp_h.assign(N, nullptr);
  c->a_exp_d.assign(N, nullptr);
  c->a_tot_h.assign(N, nullptr);
  c->a_tot_d.assign(N, nullptr);
  c->a_ready.assign(N, nullptr);
  for (size_t k = 0; k < N; ++k) {
    BK_CUDA(cudaHostAlloc((void**)&c->a_desc_h[k], (size_t)p.L * sizeof(AddrDesc), fl));
    BK_CUDA(cudaHostAlloc((void**)&c->a_exp_h[k], std::max<uint64_t>(p.exp_cap, 64), fl));
    BK_CUDA(cudaHostAlloc((void**)&c->a_tot_h[k], 64, fl));
    BK_CUDA(cudaHostGetDevicePointer((void**)&c->a_desc_d[k], c->a_desc_h[k], 0));
    BK_CUDA(cudaHostGetDevicePointer((void**)&c->a_exp_d[k], c->a_exp_h[k], 0));
    BK_CUDA(cudaHostGetDevicePointer((void**)&c->a_tot_d[k], c->a_tot_h[k], 0));
    BK_CUDA(cudaEventCreateWithFlags(&c->a_ready[k], cudaEventDisableTiming));
  }
  c->a_L = p.L;
  c->a_exp_cap = p.exp_cap;
  return BK_OK;
}

// Stage 1 of chunk i on the GPU (s_asm): lane plan, then every lane's element addresses (from the
// access spec, or the caller's generator), pattern recognition, descriptors + explicit addresses into
// the slot's pinned host buffers; a_ready[slot] marks them complete (P:629-631 signal_addrReady).
static int addr_issue(bk_ctx* c, const Plan& p, size_t i) {
  const size_t k = i % c->cfg.n_slots;
  Slot& s = c->slots[k];
  const Chunk ch = chunk_of(c, p, i);
  Access a = p.a;
  a.rec_size = c->off ? 0 : c->cfg.record_size;
  cudaStream_t st = c->s_asm;
  if (s.used) BK_CUDA(cudaStreamWaitEvent(st, s.freed, 0));   // chunk i-N no longer reads the slot
  BK_DELAY(st);
  BK_PROF(kStAddrgen, st, true);
  if (c->off && ch.hi > ch.lo) {
    BK_CUDA(cudaMemcpyAsync(s.meta, c->off + ch.lo, (ch.hi - ch.lo) * 8, cudaMemcpyHostToDevice, st));
    c->st.bytes_meta += (ch.hi - ch.lo) * 8;
  }
  launch_addrgen(ch, a, s.meta, s.lanes, s.tileK, s.tile_base, p.stage_cap, c->d_err,
                 p.user_addr ? c->d_ctr + 7 : c->d_ctr + 0, st);
  c->n_launch += 3;
  if (p.user_addr) {   // the caller's generator writes the addresses, within each lane's capacity
    launch_lane_bases(ch.L, s.lanes, p.elem, s.ucount, s.ubase, st);
    BK_CUDA(cudaMemsetAsync(s.ucount, 0, (size_t)ch.L * 4, st));
    bk_addr_view v{};
    v.struct_size = sizeof(bk_addr_view);
    v.lanes = ch.L;
    v.chunk_index = i;
    v.n_chunks = p.bounds.size() - 1;
    v.first_record = ch.lo;
    v.n_records = ch.hi - ch.lo;
    v.lane_desc = reinterpret_cast<const bk_lane*>(s.lanes);
    v.offsets = c->off ? s.meta : nullptr;
    v.end_offset = ch.end_byte;
    v.addr = s.uaddr;
    v.addr_base = s.ubase;
    v.addr_count = s.ucount;
    v.elem_bytes = p.elem;
    const int r = c->a_gen(&v, (void*)st, c->a_gen_user);
    if (r) return fail(BK_E_INVAL, "address generator returned %d for chunk %zu", r, i);
    c->n_launch += 2;
  }
  launch_addr_stage1(ch, a, s.meta, s.lanes, s.tileK, p.elem, 8, 4, !(c->cfg.flags & BK_FLAG_NO_PATTERNS),
                     p.user_addr ? s.uaddr : nullptr, s.ubase, s.ucount, c->a_desc_d[k], s.ecount, s.epos, s.exp,
                     c->a_exp_d[k], c->a_tot_d[k], st);
  c->n_launch += 4;
  if (p.user_addr) {   // lane sizes are the generated counts: tile bases again
    launch_tile_scan(s.tileK, ch.ntiles, s.tile_base, p.stage_cap, c->d_err, c->d_ctr + 0, st);
    c->n_launch += 1;
  }
  BK_PROF(kStAddrgen, st, false);
  BK_CUDA(cudaEventRecord(c->a_ready[k], st));
  return BK_OK;
}

// Chunk i: stage 1 is issued one chunk ahead (the GPU generates chunk i+1's addresses while the host
// assembles chunk i), the host waits for chunk i's addresses (P:691 wait_addrReady), assembles the
// lanes from patterns / explicit addresses into pinned staging, one DMA.
int stage_chunk_addr(bk_ctx* c, const Plan& p, size_t i, Slot& s) {
  const size_t C = p.bounds.size() - 1;
  while (c->addr_next < C && c->addr_next <= i + 1) {
    const int rc = addr_issue(c, p, c->addr_next++);
    if (rc) return rc;
  }
  const size_t k = i % c->cfg.n_slots;
  const Chunk ch = chunk_of(c, p, i);
  const auto t0 = std::chrono::steady_clock::now();
  BK_CUDA(cudaEventSynchronize(c->a_ready[k]));
  const auto t1 = std::chrono::steady_clock::now();
  c->st.ms_addr_wait += std::chrono::duration<double, std::milli>(t1 - t0).count();
  const size_t hs = c->h_next++ % c->hstage.size();
  if (c->h_used[hs]) BK_CUDA(cudaEventSynchronize(c->h_done[hs]));
  if (c->cfg.flags & BK_FLAG_TEST_DELAYS) std::this_thread::sleep_for(std::chrono::microseconds(test_rand(c) % 200));
  const uint64_t n_exp = *reinterpret_cast<volatile uint64_t*>(c->a_tot_h[k]);
  HostData d{c->host, c->off, c->n, c->nbytes, c->cfg.record_size};
  const auto t2 = std::chrono::steady_clock::now();
  const uint64_t size = host_assemble_addr(*c->pool, d, ch.L, p.elem, c->a_desc_h[k], c->a_exp_h[k], n_exp,
                                           c->hstage[hs], p.stage_cap, c->a_epos, c->a_tbase);
  c->st.ms_cpu_gather += std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t2).count();
  if (size == UINT64_MAX) return fail(BK_E_RANGE, "address-mode chunk exceeds its slot (internal bound violated)");
  if (size == UINT64_MAX - 1)
    return fail(BK_E_INVAL, "chunk %zu: an element address lies outside the data set (or a count exceeds its lane)", i);
  uint64_t pl = 0, na = 0;
  for (uint32_t t = 0; t < ch.L; ++t) {
    pl += c->a_desc_h[k][t].p > 0;
    na += c->a_desc_h[k][t].count;
  }
  c->st.n_addr_lanes += ch.L;
  c->st.n_pattern_lanes += pl;
  c->st.n_addresses += na;
  c->st.n_explicit_addr += n_exp;
  c->st.bytes_addr += (uint64_t)ch.L * sizeof(AddrDesc) + n_exp * 8 + 8;
  c->st.n_chunks_cpu += 1;
  if (s.used) BK_CUDA(cudaStreamWaitEvent(c->s_copy, s.freed, 0));
  BK_CUDA(cudaStreamWaitEvent(c->s_copy, c->a_ready[k], 0));   // tile bases of this chunk are on the device
  BK_DELAY(c->s_copy);
  BK_PROF(kStH2D, c->s_copy, true);
  if (size) BK_CUDA(cudaMemcpyAsync(s.stage, c->hstage[hs], size, cudaMemcpyHostToDevice, c->s_copy));
  BK_CUDA(cudaEventRecord(c->h_done[hs], c->s_copy));
  c->h_used[hs] = true;
  BK_PROF(kStH2D, c->s_copy, false);
  c->st.bytes_h2d += size;
  c->st.bytes_accessed += ch.accessed;
  BK_CUDA(cudaEventRecord(s.ready, c->s_copy));
  s.used = true;
  return BK_OK;
}

// Stages 1-3 of chunk i into slot s (ZC: a staging stream; DENSE: s_copy + s_asm); records s.ready.
int stage_chunk(bk_ctx* c, const Plan& p, size_t i, Slot& s) {
  const Chunk ch = chunk_of(c, p, i);
  Access a = p.a;
  a.rec_size = c->off ? 0 : c->cfg.record_size;
  if (p.zero_copy) {
    // ZC: stages 1-3 of slot k's chunks on slot k's own staging stream, so consecutive zero-copy
    // gathers overlap (one gather's ramp-up and tail hide under the next one's transfer).
    // HYBRID: the zero-copy chunks on one stream of their own (s_asm), so a gather shares the link
    // with the DMAs of host-packed chunks instead of queueing behind them on s_copy — the
    // request-bound gather leaves wire capacity the DMAs use (grep +3-10% on two boxes,
    // profiles/r02_hybrid_streams.md) — while zero-copy gathers still run one at a time (several at
    // once slowed a 2-packer rank by 10%). Chunks then become ready out of order, which every
    // compute path allows (per-chunk outputs are indexed by chunk; ordered computes wait for each
    // chunk's ready event in chunk order).
    cudaStream_t ss = p.mode == BK_GATHER_HYBRID ? c->s_asm : c->s_stage[i % c->cfg.n_slots];
    // two descriptor sets: stage 1 of this chunk writes the set chunk i-2N used, whose compute
    // ended before chunk i-N's gather started (that gather waited for it, earlier on this stream)
    const int set = p.desc_sets == 2 ? (int)((i / c->cfg.n_slots) & 1) : 0;
    s.meta = s.meta_set[set];
    s.lanes = s.lanes_set[set];
    s.tileK = s.tileK_set[set];
    s.tile_base = s.tile_base_set[set];
    const bool early = p.desc_sets == 2;   // stage 1 need not wait for the slot
    if (s.used && !early) BK_CUDA(cudaStreamWaitEvent(ss, s.freed, 0));
    BK_DELAY(ss);
    // whole variable-length records: stage 1 reads the offsets zero-copy itself (no DMA in the chain)
    const bool meta_zc = a.whole && c->off && c->off_dev;
    BK_PROF(kStH2D, ss, true);
    if (c->off && ch.hi > ch.lo) {
      if (!meta_zc)
        BK_CUDA(cudaMemcpyAsync(s.meta, c->off + ch.lo, (ch.hi - ch.lo) * 8, cudaMemcpyHostToDevice, ss));
      c->st.bytes_meta += (ch.hi - ch.lo) * 8;
    }
    BK_PROF(kStH2D, ss, false);
    BK_PROF(kStAddrgen, ss, true);
    launch_addrgen(ch, a, s.meta, s.lanes, s.tileK, s.tile_base, p.stage_cap, c->d_err, c->d_ctr + 0, ss,
                   meta_zc ? c->off_dev + ch.lo : nullptr);
    BK_PROF(kStAddrgen, ss, false);
    if (s.used && early) BK_CUDA(cudaStreamWaitEvent(ss, s.freed, 0));   // the stage buffer
    BK_DELAY(ss);
    BK_PROF(kStGather, ss, true);
    if (p.mode == BK_GATHER_HYBRID) BK_CUDA(cudaEventRecord(s.zt0, ss));
    Chunk gch = ch;   // readable source: the registered data set
    gch.guard_lo = ch.base_byte;
    gch.guard_hi = c->nbytes - ch.base_byte;
    launch_gather(gch, a, c->host_dev + ch.base_byte, s.meta, s.lanes, s.tile_base, s.stage, p.stage_cap, 1, ss);
    if (p.mode == BK_GATHER_HYBRID) BK_CUDA(cudaEventRecord(s.zt1, ss));
    BK_PROF(kStGather, ss, false);
    c->n_launch += 3;
    c->st.bytes_h2d += ch.accessed;
    c->st.n_chunks_zc += 1;
    c->st.bytes_zc += ch.accessed;
    c->st.records_zc += ch.hi - ch.lo;
    BK_CUDA(cudaEventRecord(s.ready, ss));
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
  if (!p.zero_copy) BK_CUDA(cudaEventRecord(s.ready, c->s_asm));
  s.used = true;
  return BK_OK;
}

void note_plan(bk_ctx* c, const Plan& p) {
  c->st.gather_mode = (uint32_t)p.mode;
  c->st.addr_elem_bytes = p.elem;
  c->st.chunk_budget = p.budget;
  c->st.lanes = p.L;
}

int check_err(bk_ctx* c) {  // after end_host: the error bits arrived with the run's tail copy
  const int herr = (int)(uint32_t)c->h_ctr[8];
  if (herr & kErrStageOverflow) return fail(BK_E_RANGE, "staged chunk exceeded its slot (internal bound violated)");
  if (herr & kErrKeyRange) return fail(BK_E_INVAL, "a group-by key is >= G");
  if (herr & kErrTableFull) return fail(BK_E_CAPACITY, "hash table full (word count / k-mers); raise table_slots");
  if (herr & kErrWordTooLong) return fail(BK_E_RANGE, "a word is longer than 2^24 bytes or offset >= 2^40");
  if (herr & kErrFusedTimeout) return fail(BK_E_CUDA, "persistent kernel: a loader/consumer wait timed out");
  return BK_OK;
}

// ---- the pipeline driver: chunk i goes through slot i % N; stages 1-3 on the copy/assembly
// streams, stage 4 on the compute stream. `concurrent`: the kernel's updates commute (atomic
// aggregation), so chunk i's compute runs on slot stream i % N and may overlap chunk i-1's;
// otherwise (grep's ordered output) every compute is serialised on s_comp.

int begin_run(bk_ctx* c, void* stream) {
  BK_CUDA(cudaSetDevice(c->cfg.device));
  c->st.graph_issue = 0;   // the baselines issue eagerly
  if (int rt = trace_begin(c)) return rt;
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
  c->st.n_chunks_zc = c->st.bytes_zc = c->st.records_zc = 0;
  c->st.bytes_addr = c->st.n_addr_lanes = c->st.n_pattern_lanes = c->st.n_addresses = c->st.n_explicit_addr = 0;
  c->st.ms_addr_wait = 0;
  return BK_OK;
}

// Per-stage busy sums and, from (stage, begin, end) intervals relative to the run start, the union
// of transfer intervals, the union of compute intervals and their overlap (the north_star's
// copy/compute overlap). Intervals come from BK_FLAG_PROFILE's event pairs (eager issue) or from
// BK_FLAG_TRACE's CUPTI records (the graph-replayed pipeline as timed).
struct Interval { int stage; double b, e; };

static void interval_stats(bk_ctx* c, const std::vector<Interval>& iv) {
  double acc[kNStages] = {};
  uint64_t cnt[kNStages] = {};
  std::vector<std::pair<double, double>> xfer, comp;
  // BK_TIMELINE=<path>: append every interval of the run as CSV (stage ids as kSt* in runtime.cuh)
  const char* tl_path = getenv("BK_TIMELINE");
  FILE* tl = tl_path ? fopen(tl_path, "a") : nullptr;
  if (tl) fprintf(tl, "# run\n");
  for (const auto& x : iv) {
    if (tl) fprintf(tl, "%d,%.4f,%.4f\n", x.stage, x.b, x.e);
    acc[x.stage] += x.e - x.b;
    cnt[x.stage] += 1;
    if (x.stage == kStH2D || x.stage == kStGather || x.stage == kStD2H) xfer.emplace_back(x.b, x.e);
    if (x.stage == kStCompute) comp.emplace_back(x.b, x.e);
  }
  if (tl) fclose(tl);
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
  c->st.ms_zc = acc[kStGather];
  c->st.n_zc = cnt[kStGather];
  c->st.ms_relayout = acc[kStRelayout];
  c->st.n_relayout = cnt[kStRelayout];
  c->st.ms_d2h = acc[kStD2H];
  c->st.n_d2h = cnt[kStD2H];
  c->st.ms_xfer_busy = bx;
  c->st.ms_compute_busy = bc;
  c->st.ms_overlap = ov;
}

int stage_stats(bk_ctx* c) {
  std::vector<Interval> iv;
  for (size_t i = 0; i + 1 < c->prof_used + 1 && i < c->prof_used; i += 2) {
    float e = 0, b0 = 0;
    BK_CUDA(cudaEventElapsedTime(&e, c->prof[i], c->prof[i + 1]));
    BK_CUDA(cudaEventElapsedTime(&b0, c->t_begin, c->prof[i]));
    iv.push_back({c->prof_stage[i / 2], b0, b0 + e});
  }
  interval_stats(c, iv);
  return BK_OK;
}

// BK_FLAG_TRACE: stage of a traced kernel / copy, by the kernel's (mangled) name; -1 = not a stage
// (memsets, finalize / compaction kernels, test spins)
static int trace_stage(const trace::Rec& r) {
  if (r.kind == trace::Rec::kMemcpy) return r.copy_kind == 1 ? kStH2D : r.copy_kind == 2 ? kStD2H : -1;
  if (r.kind != trace::Rec::kKernel) return -1;
  const std::string& n = r.name;
  auto has = [&](const char* x) { return n.find(x) != std::string::npos; };
  if (has("k_gather_")) return has("ILb1E") ? kStGather : kStRelayout;   // <kHost = true>: zero-copy
  if (has("k_wc_fused")) return kStGather;                                 // stages 1-4 in one kernel
  if (has("k_lane_first") || has("k_addrgen") || has("k_tile_scan") || has("k_addr_") || has("k_lane_caps"))
    return kStAddrgen;
  if (has("compact") || has("k_grep_order") || has("k_merge") || has("k_spin")) return -1;
  return kStCompute;
}

int trace_begin(bk_ctx* c) {
  c->tracing = false;
  if (!(c->cfg.flags & BK_FLAG_TRACE)) return BK_OK;
  if (trace::begin(&c->trace_recs)) return fail(BK_E_UNSUPPORTED, "BK_FLAG_TRACE: libcupti not available");
  c->tracing = true;
  return BK_OK;
}

static void trace_finish(bk_ctx* c) {
  trace::end();
  c->tracing = false;
  std::vector<Interval> iv;
  uint64_t t0 = UINT64_MAX, t1 = 0;
  for (const auto& r : c->trace_recs) {
    t0 = std::min(t0, r.start);
    t1 = std::max(t1, r.end);
  }
  for (const auto& r : c->trace_recs) {
    const int stg = trace_stage(r);
    if (stg >= 0) iv.push_back({stg, (r.start - t0) * 1e-6, (r.end - t0) * 1e-6});
  }
  interval_stats(c, iv);
  c->st.ms_trace_span = t1 > t0 ? (t1 - t0) * 1e-6 : 0.0;
  c->st.n_trace_records = c->trace_recs.size();
}

int end_run(bk_ctx* c, void* stream) { return end_host(c, stream); }

// ---- run_device: fork/join all streams around a pipeline; capture it as a CUDA graph once per key
std::vector<cudaStream_t> side_streams(bk_ctx* c) {
  std::vector<cudaStream_t> v{c->s_copy, c->s_asm, c->s_d2h};
  for (auto st : c->s_slot) v.push_back(st);
  for (auto st : c->s_stage) v.push_back(st);
  return v;
}

int device_begin(bk_ctx* c) {
  BK_CUDA(cudaMemsetAsync(c->d_err, 0, sizeof(int), c->s_comp));
  BK_CUDA(cudaMemsetAsync(c->d_ctr, 0, 8 * sizeof(unsigned long long), c->s_comp));
  BK_CUDA(cudaEventRecord(c->ev_fork, c->s_comp));
  for (auto st : side_streams(c)) BK_CUDA(cudaStreamWaitEvent(st, c->ev_fork, 0));
  // test delays: s_comp lags the side streams by ~2 ms here, so a chunk stage that does not wait
  // for the driver's setup on s_comp (centroids, memsets) reads it uninitialised
  if (c->cfg.flags & BK_FLAG_TEST_DELAYS) launch_spin(4000000, c->s_comp);
  return BK_OK;
}

// Work a kernel driver enqueues on s_comp after device_begin (centroid upload, aggregate / table /
// cursor memsets) must precede every chunk's compute: the pipeline makes the per-slot compute streams
// wait for s_comp again before its first chunk (stages 1-3 do not read that state, so the first DMAs
// and gathers still start at once). Without it the compute streams depended only on the first fork
// (gpurun_out/r02s: eager k-means at 2.5e8 points computed its first chunks against the zeroed
// centroid buffer; graph replays had hidden the missing edge by timing).
int refork(bk_ctx* c) {
  BK_CUDA(cudaEventRecord(c->ev_fork, c->s_comp));
  for (auto st : c->s_slot) BK_CUDA(cudaStreamWaitEvent(st, c->ev_fork, 0));
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
  c->st.n_chunks_zc = c->st.bytes_zc = c->st.records_zc = 0;
  c->st.bytes_addr = c->st.n_addr_lanes = c->st.n_pattern_lanes = c->st.n_addresses = c->st.n_explicit_addr = 0;
  c->st.ms_addr_wait = 0;
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
  // the run's tail: counters + error bits into pinned memory, then ONE host sync per run
  c->h_ctr[8] = 0;
  BK_CUDA(cudaMemcpyAsync(c->h_ctr, c->d_ctr, 8 * sizeof(unsigned long long), cudaMemcpyDeviceToHost, c->s_comp));
  BK_CUDA(cudaMemcpyAsync(c->h_ctr + 8, c->d_err, sizeof(int), cudaMemcpyDeviceToHost, c->s_comp));
  BK_CUDA(cudaEventRecord(c->t_end, c->s_comp));   // outside any graph: graph event nodes carry no timestamps
  BK_CUDA(cudaEventRecord(c->ev_end, c->s_comp));
  BK_CUDA(cudaStreamWaitEvent((cudaStream_t)stream, c->ev_end, 0));
  BK_CUDA(cudaStreamSynchronize(c->s_comp));
  const unsigned long long staged = c->h_ctr[0];
  c->st.bytes_padding = staged >= c->st.bytes_accessed ? staged - c->st.bytes_accessed : 0;
  float ms = 0;
  BK_CUDA(cudaEventElapsedTime(&ms, c->t_begin, c->t_end));
  c->st.ms_device = ms;
  if (c->tracing) {
    trace_finish(c);
  } else {
    int rc = stage_stats(c);
    if (rc) return rc;
  }
  return check_err(c);
}

// Runs `enqueue` (which issues one whole pipeline on the context's streams) ordered after `stream`.
// ZC / DENSE pipelines are fully static for a given key, so the first run captures them as a
// CUDA graph and later runs replay it (BK_FLAG_NO_GRAPH forces eager issue).

void drop_graphs(bk_ctx* c) {
  for (auto& g : c->graphs)
    if (g.exec) cudaGraphExecDestroy(g.exec);
  c->graphs.clear();
}

bool graphable(const Plan& p) { return p.mode == BK_GATHER_ZC || p.mode == BK_GATHER_DENSE; }

std::string resident_key(const bk_ctx* c) {
  std::string k;
  char b[24];
  for (const DevBuf* d : {&c->b_table, &c->b_out1, &c->b_out2, &c->b_out3, &c->b_blk, &c->b_blk2, &c->b_blk3,
                          &c->b_agg1, &c->b_agg2, &c->b_agg3, &c->b_mu, &c->b_hist, &c->b_colpre, &c->b_totals,
                          &c->b_base, &c->b_h1, &c->b_h2, &c->b_units, &c->b_flags, &c->b_kbin}) {
    snprintf(b, sizeof b, "%llx,", (unsigned long long)(uintptr_t)d->p);
    k += b;
  }
  return k;
}


// Identity of a caller-owned buffer a captured graph bakes in (a D2H destination, a mapped result
// array): its address AND the CUDA allocation it belongs to (CU_POINTER_ATTRIBUTE_BUFFER_ID, unique
// per allocation / registration in the process). A graph whose copy targets a registration that was
// since released — or memory freed and reallocated at the same address — must never be replayed:
// the driver resolved its DMA mapping at capture (a replay after re-registration crashed in the
// driver, gpurun_out/r02f1: partition run twice on one registration). Unknown memory: address only.
std::string mem_key(const void* p) {
  using PfnPtrAttr = CUresult (*)(void*, CUpointer_attribute, CUdeviceptr);
  static PfnPtrAttr attr = [] {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    PfnPtrAttr r = nullptr;
    if (cudaGetDriverEntryPoint("cuPointerGetAttribute", &f, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      r = reinterpret_cast<PfnPtrAttr>(f);
    cudaGetLastError();
    return r;
  }();
  unsigned long long id = 0;
  if (p && attr && attr(&id, CU_POINTER_ATTRIBUTE_BUFFER_ID, (CUdeviceptr)(uintptr_t)p) != CUDA_SUCCESS) id = 0;
  char b[48];
  snprintf(b, sizeof b, "%llx#%llx", (unsigned long long)(uintptr_t)p, id);
  return b;
}

// The caller's per-record outputs (partition records, k-means cid, k-mer arrays) are written by DMA,
// so they must be page-locked while the run copies into them. By default they are registered for
// the run only (release_run_outputs at the end of bk_run); with BK_FLAG_KEEP_OUTPUTS_PINNED the
// registration is cached across runs (at most four arrays, oldest released first) and dropped by
// bk_unpin_outputs / bk_destroy — the caller then keeps those arrays alive until one of them.
int ensure_out_pinned(bk_ctx* c, void* ptr, uint64_t bytes) {
  if (!bytes) return BK_OK;
  const bool keep = (c->cfg.flags & BK_FLAG_KEEP_OUTPUTS_PINNED) != 0;
  for (auto& e : c->out_pinned)
    if (e.first == ptr && e.second == bytes) return BK_OK;
  for (auto& e : c->out_pinned_run)
    if (e.first == ptr && e.second >= bytes) return BK_OK;
  cudaPointerAttributes at;
  if (cudaPointerGetAttributes(&at, ptr) == cudaSuccess && at.type != cudaMemoryTypeUnregistered)
    return BK_OK;   // device / managed memory, the caller's own pinned memory, or still registered by us
  cudaGetLastError();
  if (keep && c->out_pinned.size() >= 8) {
    cudaHostUnregister(c->out_pinned.front().first);
    c->out_pinned.erase(c->out_pinned.begin());
  }
  BK_CUDA(cudaHostRegister(ptr, bytes, cudaHostRegisterPortable | cudaHostRegisterMapped));
  (keep ? c->out_pinned : c->out_pinned_run).emplace_back(ptr, bytes);
  return BK_OK;
}

// A pointer kernels may store results through: device / managed memory as is, pinned host memory
// through its mapped alias (kernel stores travel over PCIe, overlapping the kernel), host memory the
// caller lets the context keep pinned (BK_FLAG_KEEP_OUTPUTS_PINNED: registered once); otherwise
// nullptr (the caller stages the results in HBM and copies them after the run).
void* out_kernel_ptr(bk_ctx* c, void* ptr, uint64_t bytes) {
  if (!ptr || !bytes) return nullptr;
  cudaPointerAttributes at;
  if (cudaPointerGetAttributes(&at, ptr) != cudaSuccess) {
    cudaGetLastError();
    return nullptr;
  }
  if (at.type == cudaMemoryTypeDevice || at.type == cudaMemoryTypeManaged) return ptr;
  if (at.type == cudaMemoryTypeUnregistered) {
    if (!(c->cfg.flags & BK_FLAG_KEEP_OUTPUTS_PINNED) || ensure_out_pinned(c, ptr, bytes)) {
      cudaGetLastError();
      return nullptr;
    }
  }
  // pinned host memory: both ends of the range must be mapped, at the same distance on the device
  // (a registration covers whole pages, so an array can start inside another array's registered page
  // and run past it; kernels would then store through an unmapped address)
  uint8_t* last = static_cast<uint8_t*>(ptr) + bytes - 1;
  cudaPointerAttributes at_last;
  void *d = nullptr, *d_last = nullptr;
  if (cudaPointerGetAttributes(&at_last, last) != cudaSuccess || at_last.type != cudaMemoryTypeHost ||
      cudaHostGetDevicePointer(&d, ptr, 0) != cudaSuccess || cudaHostGetDevicePointer(&d_last, last, 0) != cudaSuccess ||
      static_cast<uint8_t*>(d_last) - static_cast<uint8_t*>(d) != (ptrdiff_t)(bytes - 1)) {
    cudaGetLastError();
    return nullptr;
  }
  return d;
}

// End of every bk_run (after all its copies completed or were drained): release this run's output
// registrations.
void release_run_outputs(bk_ctx* c) {
  for (auto& e : c->out_pinned_run) cudaHostUnregister(e.first);
  c->out_pinned_run.clear();
  cudaGetLastError();
}

void release_kept_outputs(bk_ctx* c) {
  for (auto& e : c->out_pinned) cudaHostUnregister(e.first);
  c->out_pinned.clear();
  cudaGetLastError();
}

void unregister(bk_ctx* c) {
  if (c->pinned_data && c->host) cudaHostUnregister((void*)c->host);
  if (c->pinned_off && c->off) cudaHostUnregister((void*)c->off);
  c->pinned_data = c->pinned_off = c->registered = false;
  c->host = nullptr;
  c->off = nullptr;
  c->host_dev = nullptr;
  c->off_dev = nullptr;
  c->n = c->nbytes = 0;
}


}  // namespace rt
}  // namespace bk
