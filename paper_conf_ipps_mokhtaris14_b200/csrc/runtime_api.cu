// runtime_api.cu — the C ABI of include/bk.h: context creation (streams, events, window), registration
// (validate offsets once, pin once), run dispatch by kernel id, statistics, destruction.
#include "runtime.cuh"

namespace bk {
namespace rt {

namespace {
thread_local std::string g_last_error;
}  // namespace

int fail(int code, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  g_last_error = buf;
  return code;
}

const char* last_error() { return g_last_error.c_str(); }

}  // namespace rt
}  // namespace bk

using namespace bk;
using namespace bk::rt;

// After a failed run: wait for everything already queued on the context's streams (no copy may
// still target the caller's buffers, no kernel may still use the slots) and clear the error state.
static void drain(bk_ctx* c) {
  if (c->tracing) {   // a failed traced run: stop collecting
    bk::trace::end();
    c->tracing = false;
  }
  for (cudaStream_t st : {c->s_copy, c->s_asm, c->s_comp, c->s_d2h})
    if (st) cudaStreamSynchronize(st);
  for (auto st : c->s_slot) cudaStreamSynchronize(st);
  for (auto st : c->s_stage) cudaStreamSynchronize(st);
  cudaGetLastError();
}

// Selects the context's device for the duration of an API call and restores the caller's current
// device on return (a process may drive contexts on several GPUs from one thread).
struct DeviceGuard {
  int prev = -1;
  bool ok = false;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
    ok = cudaSetDevice(dev) == cudaSuccess;
    cudaGetLastError();
  }
  ~DeviceGuard() {
    if (prev >= 0) cudaSetDevice(prev);
    cudaGetLastError();
  }
  DeviceGuard(const DeviceGuard&) = delete;
  DeviceGuard& operator=(const DeviceGuard&) = delete;
};

// struct_size of the in/out struct bk_run expects for each kernel id (0: unknown id)
static uint32_t out_size(int kernel_id) {
  switch (kernel_id) {
    case BK_K_WORDCOUNT: return sizeof(bk_out_wordcount);
    case BK_K_GREP: return sizeof(bk_out_grep);
    case BK_K_KMEANS: return sizeof(bk_out_kmeans);
    case BK_K_PARTITION: return sizeof(bk_out_partition);
    case BK_K_GROUPBY: return sizeof(bk_out_groupby);
    case BK_K_KMER: return sizeof(bk_out_kmer);
    case BK_K_LAYOUT_DUMP: return sizeof(bk_out_layout);
    case BK_K_PATTERN_STATS: return sizeof(bk_out_pattern);
    default: return 0;
  }
}

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

const char* bk_last_error(void) { return bk::rt::last_error(); }

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
  DeviceGuard dg(c->cfg.device);
  if (!dg.ok) return cleanup(fail(BK_E_CUDA, "cudaSetDevice"));
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
  if (cudaHostAlloc(&c->h_ctr, 9 * sizeof(unsigned long long), cudaHostAllocDefault) != cudaSuccess)
    return cleanup(fail(BK_E_NOMEM, "cudaHostAlloc counters"));
  c->slots.resize(c->cfg.n_slots);
  if (cudaStreamCreateWithFlags(&c->s_d2h, cudaStreamNonBlocking) != cudaSuccess) return cleanup(fail(BK_E_CUDA, "d2h stream"));
  if (configure_partition_kernels() != cudaSuccess || configure_baseline_kernels() != cudaSuccess ||
      configure_kmer_kernels() != cudaSuccess)
    return cleanup(fail(BK_E_CUDA, "cudaFuncSetAttribute"));
  if (cudaEventCreateWithFlags(&c->ev_fork, cudaEventDisableTiming) != cudaSuccess ||
      cudaEventCreateWithFlags(&c->ev_fused, cudaEventDisableTiming) != cudaSuccess)
    return cleanup(fail(BK_E_CUDA, "events"));
  c->ev_join.assign(3 + 2 * c->cfg.n_slots, nullptr);
  for (auto& e : c->ev_join)
    if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) return cleanup(fail(BK_E_CUDA, "events"));
  c->ev_part.assign(c->cfg.n_slots, nullptr);
  for (auto& e : c->ev_part)
    if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) return cleanup(fail(BK_E_CUDA, "events"));
  c->s_slot.assign(c->cfg.n_slots, nullptr);
  for (auto& st : c->s_slot)
    if (cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking) != cudaSuccess) return cleanup(fail(BK_E_CUDA, "slot streams"));
  c->s_stage.assign(c->cfg.n_slots, nullptr);
  for (auto& st : c->s_stage)
    if (cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking) != cudaSuccess) return cleanup(fail(BK_E_CUDA, "slot streams"));
  for (auto& s : c->slots) {
    if (cudaEventCreateWithFlags(&s.copied, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&s.ready, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&s.freed, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreate(&s.zt0) != cudaSuccess || cudaEventCreate(&s.zt1) != cudaSuccess)
      return cleanup(fail(BK_E_CUDA, "slot events"));
  }
  c->st.struct_size = sizeof(bk_stats);
  c->st.n_slots = c->cfg.n_slots;
  c->st.slot_bytes = c->cfg.window_bytes / c->cfg.n_slots;
  *out_ctx = c;
  return BK_OK;
}

int bk_register_segments(bk_ctx* c, const void* host_ptr, uint64_t nbytes, const uint64_t* off, uint64_t n) {
  NvtxRange nv("bk_register_segments");
  if (!c) return fail(BK_E_INVAL, "NULL ctx");
  if (!host_ptr && nbytes) return fail(BK_E_INVAL, "NULL host_ptr");
  const auto t0 = std::chrono::steady_clock::now();
  DeviceGuard dg(c->cfg.device);
  if (!dg.ok) return fail(BK_E_CUDA, "cudaSetDevice");
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
      // read-only where supported (libbk never writes the registered data set) and only
      // when the range owns whole pages: a read-only registration of a page that also holds other
      // objects makes every later registration touching that page fail (measured: offsets arrays
      // and output arrays from the same heap pages -> cudaErrorInvalidValue)
      int ro = 0;
      cudaDeviceGetAttribute(&ro, cudaDevAttrHostRegisterReadOnlySupported, c->cfg.device);
      const uintptr_t pg = 4096;
      if ((uintptr_t)host_ptr % pg || nbytes % pg) ro = 0;
      const unsigned fl = cudaHostRegisterMapped | cudaHostRegisterPortable | (ro ? cudaHostRegisterReadOnly : 0u);
      cudaError_t e = cudaHostRegister((void*)host_ptr, nbytes, fl);
      if (e != cudaSuccess && ro) {   // some platforms advertise but refuse it: plain mapped registration
        cudaGetLastError();
        e = cudaHostRegister((void*)host_ptr, nbytes, cudaHostRegisterMapped | cudaHostRegisterPortable);
      }
      c->registered_ro = e == cudaSuccess && ro;
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
    c->host = (const uint8_t*)host_ptr;   // from here on unregister() releases what was pinned
  }
  if (off && n) {
    if (is_pinned(off)) {
      c->pinned_off = false;
    } else {
      cudaError_t e = cudaHostRegister((void*)off, n * 8, cudaHostRegisterMapped | cudaHostRegisterPortable);
      if (e != cudaSuccess) {
        unregister(c);   // do not leak the data set's pinning on a failed registration
        return fail(BK_E_CUDA, "cudaHostRegister(offsets): %s", cudaGetErrorString(e));
      }
      c->pinned_off = true;
    }
    void* odev = nullptr;  // caller-pinned offsets may be unmapped: then stage 1 DMAs them instead
    c->off_dev = cudaHostGetDevicePointer(&odev, (void*)off, 0) == cudaSuccess ? (const uint64_t*)odev : nullptr;
    cudaGetLastError();
  }
  c->host = (const uint8_t*)host_ptr;
  c->nbytes = nbytes;
  c->off = off;
  c->n = n;
  c->registered = true;
  c->plan_cache.clear();
  c->units_key.clear();
  c->batch_key.clear();
  c->hy_t_zc_ms = c->hy_t_cpu_ms = 0;
  drop_graphs(c);
  c->st.ms_register = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  return BK_OK;
}

int bk_run(bk_ctx* c, int kernel_id, void* stream, void* out) {
  if (!c || !out) return fail(BK_E_INVAL, "NULL argument");
  if (!c->registered) return fail(BK_E_STATE, "bk_run before bk_register_segments");
  const bk_out_header* h = (const bk_out_header*)out;
  if (h->kernel_id != kernel_id) return fail(BK_E_INVAL, "out->kernel_id %d != %d", h->kernel_id, kernel_id);
  const uint32_t want = out_size(kernel_id);
  if (!want) return fail(BK_E_UNSUPPORTED, "unknown kernel_id %d", kernel_id);
  if (h->struct_size != want) return fail(BK_E_INVAL, "out struct_size %u != %u for kernel %d", h->struct_size, want, kernel_id);
  DeviceGuard dg(c->cfg.device);   // every allocation and launch of this run lands on the context's GPU
  if (!dg.ok) return fail(BK_E_CUDA, "cudaSetDevice(%d)", c->cfg.device);
  static const char* const kNames[] = {"?", "wordcount", "grep", "kmeans", "partition", "groupby", "kmer"};
  NvtxRange nv("bk_run.%s", kernel_id >= 1 && kernel_id <= 6 ? kNames[kernel_id]
                             : kernel_id == BK_K_LAYOUT_DUMP ? "layout" : "pattern");
  const auto t0 = std::chrono::steady_clock::now();
  int rc;
  if (c->cfg.flags & (BK_FLAG_BASELINE_DBUF | BK_FLAG_BASELINE_SBUF)) {
    rc = run_dbuf(c, kernel_id, out, stream);
    if (rc) drain(c);
    release_run_outputs(c);
    if (rc) return rc;
    c->st.kernel_launches = (uint64_t)c->n_launch;
    c->st.ms_run = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    return BK_OK;
  }
  switch (kernel_id) {
    case BK_K_WORDCOUNT:
      rc = run_wordcount(c, (bk_out_wordcount*)out, stream);
      break;
    case BK_K_GREP:
      rc = run_grep(c, (bk_out_grep*)out, stream);
      break;
    case BK_K_KMEANS:
      rc = run_kmeans(c, (bk_out_kmeans*)out, stream);
      break;
    case BK_K_GROUPBY:
      rc = run_groupby(c, (bk_out_groupby*)out, stream);
      break;
    case BK_K_KMER:
      rc = run_kmer(c, (bk_out_kmer*)out, stream);
      break;
    case BK_K_PATTERN_STATS:
      rc = run_pattern(c, (bk_out_pattern*)out, stream);
      break;
    case BK_K_LAYOUT_DUMP:
      rc = run_layout(c, (bk_out_layout*)out, stream);
      break;
    case BK_K_PARTITION:
      rc = run_partition(c, (bk_out_partition*)out, stream);
      break;
    default:
      return fail(BK_E_UNSUPPORTED, "unknown kernel_id %d", kernel_id);
  }
  if (rc) drain(c);   // leave the context usable
  release_run_outputs(c);
  if (rc) return rc;
  c->st.kernel_launches = (uint64_t)c->n_launch;
  c->st.ms_run = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  return BK_OK;
}

int bk_run_user(bk_ctx* c, const bk_access* a, bk_chunk_fn fn, void* user, void* stream) {
  NvtxRange nv("bk_run_user");
  if (!c || !a || !fn) return fail(BK_E_INVAL, "NULL argument");
  if (a->struct_size != sizeof(bk_access)) return fail(BK_E_INVAL, "bk_access size");
  if (!c->registered) return fail(BK_E_STATE, "bk_run_user before bk_register_segments");
  if (c->cfg.flags & (BK_FLAG_BASELINE_DBUF | BK_FLAG_BASELINE_SBUF))
    return fail(BK_E_UNSUPPORTED, "bk_run_user: no double-buffering baseline for user kernels");
  DeviceGuard dg(c->cfg.device);
  if (!dg.ok) return fail(BK_E_CUDA, "cudaSetDevice(%d)", c->cfg.device);
  const auto t0 = std::chrono::steady_clock::now();
  const int rc = run_user(c, a, fn, user, stream);
  if (rc) {
    drain(c);
    return rc;
  }
  c->st.kernel_launches = (uint64_t)c->n_launch;
  c->st.ms_run = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  return BK_OK;
}

int bk_merge_counts(bk_ctx* c, const uint64_t* rows, uint32_t n_seg, uint64_t seg_stride, const uint64_t* seg_rows,
                    uint32_t row_u64, uint32_t key_u64, uint32_t count_col, uint64_t* out, uint64_t cap,
                    uint64_t* n_out, void* stream) {
  NvtxRange nv("bk_merge_counts");
  if (!c || !n_out || (n_seg && !seg_rows)) return fail(BK_E_INVAL, "NULL argument");
  if (key_u64 == 0 || count_col < key_u64 || count_col >= row_u64 || row_u64 > 16)
    return fail(BK_E_INVAL, "need 1 <= key_u64 <= count_col < row_u64 <= 16");
  if (n_seg > 64) return fail(BK_E_INVAL, "at most 64 segments");
  uint64_t total = 0;
  for (uint32_t i = 0; i < n_seg; ++i) {
    if (seg_rows[i] > seg_stride) return fail(BK_E_INVAL, "seg_rows[%u] > seg_stride", i);
    total += seg_rows[i];
  }
  if (total && !rows) return fail(BK_E_INVAL, "NULL rows");
  if (cap && !out) return fail(BK_E_INVAL, "NULL out");
  DeviceGuard dg(c->cfg.device);
  if (!dg.ok) return fail(BK_E_CUDA, "cudaSetDevice(%d)", c->cfg.device);
  uint64_t slots = 1024;
  while (slots < 2 * total) slots <<= 1;
  BK_CUDA(c->b_mown.ensure(slots * 8));
  BK_CUDA(c->b_mcnt.ensure(slots * 8));
  BK_CUDA(c->b_mctr.ensure(16));
  cudaStream_t st = c->s_comp;
  BK_CUDA(cudaEventRecord(c->ev_begin, (cudaStream_t)stream));
  BK_CUDA(cudaStreamWaitEvent(st, c->ev_begin, 0));
  BK_CUDA(cudaMemsetAsync(c->d_err, 0, sizeof(int), st));
  BK_CUDA(launch_merge_counts(rows, n_seg, seg_stride, seg_rows, row_u64, key_u64, count_col,
                              (unsigned long long*)c->b_mown.p, (unsigned long long*)c->b_mcnt.p, slots, out, cap,
                              (unsigned long long*)c->b_mctr.p, c->d_err, st));
  BK_CUDA(cudaMemcpyAsync(c->h_ctr, c->b_mctr.p, 8, cudaMemcpyDeviceToHost, st));
  BK_CUDA(cudaMemcpyAsync(c->h_ctr + 8, c->d_err, sizeof(int), cudaMemcpyDeviceToHost, st));
  BK_CUDA(cudaEventRecord(c->ev_end, st));
  BK_CUDA(cudaStreamWaitEvent((cudaStream_t)stream, c->ev_end, 0));
  BK_CUDA(cudaStreamSynchronize(st));
  if ((int)(uint32_t)c->h_ctr[8] & kErrTableFull) return fail(BK_E_CUDA, "merge table full (internal bound violated)");
  *n_out = c->h_ctr[0];
  if (*n_out > cap) return fail(BK_E_CAPACITY, "%llu distinct keys > cap %llu", (unsigned long long)*n_out,
                                (unsigned long long)cap);
  return BK_OK;
}

int bk_unpin_outputs(bk_ctx* c) {
  if (!c) return fail(BK_E_INVAL, "NULL ctx");
  DeviceGuard dg(c->cfg.device);
  release_kept_outputs(c);
  return BK_OK;
}

int bk_run_user_addr(bk_ctx* c, const bk_access* a, bk_addr_fn gen, void* gen_user, bk_chunk_fn fn, void* user,
                     void* stream) {
  NvtxRange nv("bk_run_user_addr");
  if (!c || !a || !gen || !fn) return fail(BK_E_INVAL, "NULL argument");
  if (a->struct_size != sizeof(bk_access)) return fail(BK_E_INVAL, "bk_access size");
  if (!c->registered) return fail(BK_E_STATE, "bk_run_user_addr before bk_register_segments");
  if (c->cfg.flags & (BK_FLAG_BASELINE_DBUF | BK_FLAG_BASELINE_SBUF))
    return fail(BK_E_UNSUPPORTED, "bk_run_user_addr: no double-buffering baseline for user kernels");
  DeviceGuard dg(c->cfg.device);
  if (!dg.ok) return fail(BK_E_CUDA, "cudaSetDevice(%d)", c->cfg.device);
  const auto t0 = std::chrono::steady_clock::now();
  const int rc = run_user_addr(c, a, gen, gen_user, fn, user, stream);
  if (rc) {
    drain(c);
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

int bk_partition_materialize(const void* out_records, const uint64_t* chunk_counts, uint64_t n_chunks,
                             uint32_t n_buckets, const uint64_t* bucket_start, void* dst, uint32_t threads) {
  if (n_buckets == 0) return fail(BK_E_INVAL, "n_buckets == 0");
  if (n_chunks && n_chunks > UINT64_MAX / n_buckets) return fail(BK_E_INVAL, "n_chunks * n_buckets overflows");
  if (n_chunks && (!out_records || !chunk_counts || !dst)) return fail(BK_E_INVAL, "NULL argument");
  try {
    partition_materialize(static_cast<const uint8_t*>(out_records), chunk_counts, n_chunks, n_buckets, bucket_start,
                          static_cast<uint8_t*>(dst), threads);
  } catch (...) {
    return fail(BK_E_NOMEM, "partition_materialize: host allocation failed");
  }
  return BK_OK;
}

int bk_abi_sizes(uint32_t* sizes, int n) {
  const uint32_t v[13] = {sizeof(bk_config),     sizeof(bk_out_wordcount), sizeof(bk_out_grep),
                          sizeof(bk_out_kmeans), sizeof(bk_out_partition), sizeof(bk_out_groupby),
                          sizeof(bk_out_layout), sizeof(bk_stats),         sizeof(bk_out_pattern),
                          sizeof(bk_out_kmer),   sizeof(bk_access),        sizeof(bk_chunk_view),
                          sizeof(bk_addr_view)};
  for (int i = 0; i < n && i < 13; ++i) sizes[i] = v[i];
  return BK_ABI_VERSION;
}

int bk_destroy(bk_ctx* c) {
  if (!c) return BK_OK;
  DeviceGuard dg(c->cfg.device);
  if (c->s_comp) cudaStreamSynchronize(c->s_comp);
  if (c->s_copy) cudaStreamSynchronize(c->s_copy);
  if (c->s_asm) cudaStreamSynchronize(c->s_asm);
  for (auto st : c->s_slot)
    if (st) cudaStreamSynchronize(st);
  for (auto st : c->s_stage)
    if (st) cudaStreamSynchronize(st);
  unregister(c);
  for (auto& s : c->slots) {
    if (s.copied) cudaEventDestroy(s.copied);
    if (s.ready) cudaEventDestroy(s.ready);
    if (s.freed) cudaEventDestroy(s.freed);
    if (s.zt0) cudaEventDestroy(s.zt0);
    if (s.zt1) cudaEventDestroy(s.zt1);
  }
  for (DevBuf* b : {&c->b_table, &c->b_out1, &c->b_out2, &c->b_out3, &c->b_blk, &c->b_blk2, &c->b_blk3, &c->b_agg1, &c->b_agg2,
                    &c->b_agg3, &c->b_mu})
    b->release();
  if (c->window) cudaFree(c->window);
  if (c->d_err) cudaFree(c->d_err);
  if (c->d_ctr) cudaFree(c->d_ctr);
  if (c->d_fprof) cudaFree(c->d_fprof);
  if (c->h_ctr) cudaFreeHost(c->h_ctr);
  if (c->ev_begin) cudaEventDestroy(c->ev_begin);
  if (c->ev_end) cudaEventDestroy(c->ev_end);
  if (c->t_begin) cudaEventDestroy(c->t_begin);
  if (c->t_end) cudaEventDestroy(c->t_end);
  for (cudaEvent_t e : c->prof) cudaEventDestroy(e);
  drop_graphs(c);
  if (c->ev_fork) cudaEventDestroy(c->ev_fork);
  if (c->ev_fused) cudaEventDestroy(c->ev_fused);
  for (auto e : c->ev_join) cudaEventDestroy(e);
  if (c->h_mu) cudaFreeHost(c->h_mu);
  delete c->pool;
  if (c->s_d2h) {
    cudaStreamSynchronize(c->s_d2h);
    cudaStreamDestroy(c->s_d2h);
  }
  for (auto e : c->ev_part) cudaEventDestroy(e);
  release_run_outputs(c);
  release_kept_outputs(c);
  release_addr_side(c);
  for (DevBuf* b : {&c->b_hist, &c->b_colpre, &c->b_totals, &c->b_base, &c->b_h1, &c->b_h2, &c->b_mown, &c->b_mcnt,
                    &c->b_mctr, &c->b_units, &c->b_flags, &c->b_batch, &c->b_kbin})
    b->release();
  for (auto* h : c->hstage) cudaFreeHost(h);
  for (auto e : c->h_done) cudaEventDestroy(e);
  if (c->s_copy) cudaStreamDestroy(c->s_copy);
  if (c->s_asm) cudaStreamDestroy(c->s_asm);
  if (c->s_comp) cudaStreamDestroy(c->s_comp);
  for (auto st : c->s_slot)
    if (st) cudaStreamDestroy(st);
  for (auto st : c->s_stage)
    if (st) cudaStreamDestroy(st);
  cudaGetLastError();
  delete c;
  return BK_OK;
}

}  // extern "C"
