// trace.cpp — BK_FLAG_TRACE: per-kernel / per-copy device intervals of a run from CUPTI activity
// records (SURVEY §8(d) overlap, §5 tracing; measure overlap on the timed pass). Unlike
// BK_FLAG_PROFILE's CUDA events this keeps the CUDA-graph replay of the timed runs: CUPTI reports
// every graph kernel / memcpy node with its start and end timestamps. libcupti is loaded at run time
// (dlopen), so libbk itself needs no CUPTI to load; without it BK_FLAG_TRACE fails with
// BK_E_UNSUPPORTED.
#include "trace.h"

#include <cupti.h>
#include <dlfcn.h>

#include <cstdlib>
#include <cstring>
#include <mutex>

namespace bk {
namespace trace {
namespace {

using FnRegister = CUptiResult (*)(CUpti_BuffersCallbackRequestFunc, CUpti_BuffersCallbackCompleteFunc);
using FnEnable = CUptiResult (*)(CUpti_ActivityKind);
using FnFlush = CUptiResult (*)(uint32_t);
using FnNext = CUptiResult (*)(uint8_t*, size_t, CUpti_Activity**);

struct Api {
  bool tried = false, ok = false, registered = false;
  FnRegister reg = nullptr;
  FnEnable enable = nullptr, disable = nullptr;
  FnFlush flush = nullptr;
  FnNext next = nullptr;
};
Api g_api;
std::mutex g_mu;
std::vector<Rec>* g_sink = nullptr;
constexpr size_t kBuf = 8 << 20;

void CUPTIAPI buffer_requested(uint8_t** buffer, size_t* size, size_t* max_records) {
  *size = kBuf;
  *buffer = static_cast<uint8_t*>(aligned_alloc(8, kBuf));
  *max_records = 0;
}

void CUPTIAPI buffer_completed(CUcontext, uint32_t, uint8_t* buffer, size_t, size_t valid) {
  std::lock_guard<std::mutex> g(g_mu);
  CUpti_Activity* r = nullptr;
  while (g_api.next(buffer, valid, &r) == CUPTI_SUCCESS) {
    if (!g_sink) continue;
    Rec x{};
    if (r->kind == CUPTI_ACTIVITY_KIND_CONCURRENT_KERNEL || r->kind == CUPTI_ACTIVITY_KIND_KERNEL) {
      const auto* k = reinterpret_cast<const CUpti_ActivityKernel9*>(r);
      x.kind = Rec::kKernel;
      x.start = k->start;
      x.end = k->end;
      x.stream = k->streamId;
      x.name = k->name ? k->name : "";
    } else if (r->kind == CUPTI_ACTIVITY_KIND_MEMCPY) {
      const auto* m = reinterpret_cast<const CUpti_ActivityMemcpy6*>(r);
      x.kind = Rec::kMemcpy;
      x.copy_kind = m->copyKind;
      x.start = m->start;
      x.end = m->end;
      x.stream = m->streamId;
      x.bytes = m->bytes;
    } else if (r->kind == CUPTI_ACTIVITY_KIND_MEMSET) {
      const auto* m = reinterpret_cast<const CUpti_ActivityMemset4*>(r);
      x.kind = Rec::kMemset;
      x.start = m->start;
      x.end = m->end;
      x.stream = m->streamId;
      x.bytes = m->bytes;
    } else {
      continue;
    }
    g_sink->push_back(std::move(x));
  }
  free(buffer);
}

bool load() {
  if (g_api.tried) return g_api.ok;
  g_api.tried = true;
  void* h = nullptr;
  for (const char* n : {"libcupti.so.12", "libcupti.so", "/usr/local/cuda/lib64/libcupti.so.12",
                        "/usr/local/cuda/lib64/libcupti.so"}) {
    h = dlopen(n, RTLD_NOW | RTLD_GLOBAL);
    if (h) break;
  }
  if (!h) return false;
  g_api.reg = reinterpret_cast<FnRegister>(dlsym(h, "cuptiActivityRegisterCallbacks"));
  g_api.enable = reinterpret_cast<FnEnable>(dlsym(h, "cuptiActivityEnable"));
  g_api.disable = reinterpret_cast<FnEnable>(dlsym(h, "cuptiActivityDisable"));
  g_api.flush = reinterpret_cast<FnFlush>(dlsym(h, "cuptiActivityFlushAll"));
  g_api.next = reinterpret_cast<FnNext>(dlsym(h, "cuptiActivityGetNextRecord"));
  g_api.ok = g_api.reg && g_api.enable && g_api.disable && g_api.flush && g_api.next;
  return g_api.ok;
}

const CUpti_ActivityKind kKinds[] = {CUPTI_ACTIVITY_KIND_CONCURRENT_KERNEL, CUPTI_ACTIVITY_KIND_MEMCPY,
                                     CUPTI_ACTIVITY_KIND_MEMSET};

}  // namespace

bool available() { return load(); }

int begin(std::vector<Rec>* sink) {
  if (!load()) return -1;
  std::lock_guard<std::mutex> g(g_mu);
  if (!g_api.registered) {
    if (g_api.reg(buffer_requested, buffer_completed) != CUPTI_SUCCESS) return -2;
    g_api.registered = true;
  }
  sink->clear();
  g_sink = sink;
  for (auto k : kKinds)
    if (g_api.enable(k) != CUPTI_SUCCESS) return -3;
  return 0;
}

int end() {
  if (!g_api.ok) return -1;
  for (auto k : kKinds) g_api.disable(k);
  g_api.flush(CUPTI_ACTIVITY_FLAG_FLUSH_FORCED);
  std::lock_guard<std::mutex> g(g_mu);
  g_sink = nullptr;
  return 0;
}

}  // namespace trace
}  // namespace bk
