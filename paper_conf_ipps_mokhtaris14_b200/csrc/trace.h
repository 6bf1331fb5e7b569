// trace.h — CUPTI activity tracing of one bk_run (BK_FLAG_TRACE), see trace.cpp.
#pragma once
#include <stdint.h>

#include <string>
#include <vector>

namespace bk {
namespace trace {

struct Rec {
  enum { kKernel = 0, kMemcpy = 1, kMemset = 2 };
  int kind = 0;
  int copy_kind = 0;     // CUpti_ActivityMemcpyKind (1 = HtoD, 2 = DtoH, ...)
  uint64_t start = 0, end = 0;   // ns, device timestamps
  uint32_t stream = 0;
  uint64_t bytes = 0;
  std::string name;      // kernels: mangled name
};

bool available();
// start collecting every kernel / memcpy / memset record of this process into *sink (0 = ok)
int begin(std::vector<Rec>* sink);
// stop, flush the records into the sink (call after the traced work completed)
int end();

}  // namespace trace
}  // namespace bk
