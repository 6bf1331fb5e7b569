// host_gather.h — CPU assembly (stage 2 on the host, PAPER.md P:273-275, P:421-441, P:691-695,
// §IV.B): a persistent thread pool packs exactly the accessed bytes of a chunk into a
// pinned staging buffer in the same warp-tile layout the GPU gather produces, so stage 3 is one
// large DMA of payload bytes only. Product code (libbk): shares no code with the CPU reference under tests.
#pragma once
#include <stdint.h>

#include <atomic>
#include <condition_variable>
#include <functional>
#include <mutex>
#include <thread>
#include <vector>

#include "bk_internal.cuh"

namespace bk {

class HostPool {
 public:
  explicit HostPool(int threads);
  ~HostPool();
  int size() const { return (int)workers_.size() + 1; }
  // Runs f(tid) on every worker and on the caller (tid = size()-1); returns when all finished.
  void run(const std::function<void(int)>& f);

 private:
  void loop(int tid);
  std::vector<std::thread> workers_;
  std::mutex m_;
  std::condition_variable cv_, done_;
  std::function<void(int)> job_;
  uint64_t gen_ = 0;
  int pending_ = 0;
  bool stop_ = false;
};

struct HostData {
  const uint8_t* base;     // registered data set
  const uint64_t* off;     // record offsets (NULL = fixed records)
  uint64_t n, nbytes, rec_size;
};

// Packs chunk c into `stage` (capacity cap) with the lane rule of k_addrgen and the tile layout
// of k_gather_*; returns the staged size, or UINT64_MAX if it would exceed cap.
// Exact staged size of chunk c (512 * sum of tile word counts) under the k_addrgen lane rule.
uint64_t host_staged_size(const HostData& d, const Access& a, const Chunk& c);

uint64_t host_gather_chunk(HostPool& pool, const HostData& d, const Access& a, const Chunk& c, uint8_t* stage,
                           uint64_t cap, std::vector<uint64_t>& first_scratch, std::vector<uint64_t>& tile_scratch);

// Address mode: assemble the chunk's L lanes from their address descriptors (desc, as stage 1 wrote
// them) and the compacted explicit addresses (exp, n_exp entries) into `stage` (capacity cap), elem
// bytes per address. Returns the staged size, UINT64_MAX if it exceeds cap, UINT64_MAX - 1 if an
// address lies outside the data set or the descriptors disagree with n_exp.
uint64_t host_assemble_addr(HostPool& pool, const HostData& d, uint32_t L, uint32_t elem, const AddrDesc* desc,
                            const uint64_t* exp, uint64_t n_exp, uint8_t* stage, uint64_t cap,
                            std::vector<uint64_t>& epos, std::vector<uint64_t>& tbase);

// Single-extent access with E % 16 == 0 (host_packable): packs the chunk's accessed bytes in record
// order, E bytes per record, into dst (16-B aligned) — a sequential read of the data set and a
// sequential non-temporal write, the cheapest host gather there is. The warp-tile interleave is then
// done on the GPU (HBM -> HBM). Returns (hi - lo) * E, or UINT64_MAX if that exceeds cap.
// `grab` records per work item (0 = default); `nt`: non-temporal stores; `sink(byte_off, bytes)`, if
// set, is called by the packing thread as soon as a grab's bytes are in dst (e.g. to DMA them while
// they are still in the host's caches).
bool host_packable(const Access& a);
uint64_t host_pack_chunk(HostPool& pool, const HostData& d, const Access& a, const Chunk& c, uint8_t* dst,
                         uint64_t cap, uint64_t grab = 0, bool nt = true,
                         const std::function<void(uint64_t, uint64_t)>* sink = nullptr);

// bk_partition_materialize (include/bk.h): chunk-major bucket-sorted runs -> bucket-major order.
int partition_materialize(const uint8_t* runs, const uint64_t* counts, uint64_t n_chunks, uint32_t n_buckets,
                          const uint64_t* bucket_start, uint8_t* dst, uint32_t threads);

}  // namespace bk
