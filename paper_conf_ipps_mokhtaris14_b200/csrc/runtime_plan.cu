// runtime_plan.cu — chunk plan (greedy whole records under the budget, A3), lane-count and slot sizing,
// the per-context plan cache, and carving the window into N slots.
#include "runtime.cuh"

namespace bk {
namespace rt {

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
  const uint64_t desc = align_up(p.meta_cap * 8, kAlign) + align_up((uint64_t)p.L * sizeof(LaneDesc), kAlign) +
                        align_up(ntiles * 4, kAlign) + align_up((ntiles + 1) * 8, kAlign);
  uint64_t addr = 0;
  if (p.mode == BK_GATHER_ADDR) {
    addr = align_up(p.exp_cap, kAlign) + align_up((uint64_t)p.L * 4, kAlign) + align_up(((uint64_t)p.L + 1) * 8, kAlign);
    if (p.user_addr)
      addr += align_up(p.exp_cap, kAlign) + align_up((uint64_t)p.L * 8 + 8, kAlign) + align_up((uint64_t)p.L * 4, kAlign);
  }
  return align_up(p.raw_cap, kAlign) + align_up(p.stage_cap, kAlign) + p.desc_sets * desc + align_up(p.out_cap, kAlign) +
         addr;
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
  // DENSE: raw whole records; CPU/HYBRID with a packable access: the host-packed chunk (plan bytes
  // = accessed bytes there)
  p.raw_cap = !p.zero_copy || p.packed ? budget + 64 : 0;
  p.meta_cap = c->off ? maxrecs + 1 : 0;
  // address mode: 8 B per element address of the chunk with the most accessed bytes
  p.exp_cap = p.mode == BK_GATHER_ADDR ? (acc / std::max<uint32_t>(p.elem, 1) + 2) * 8 : 0;
}

// BK_GATHER_ADDR element size: the configured one if every accessed length is a multiple of it, else
// BK_E_INVAL; 0 = the largest power of two <= 8 dividing them (whole variable-length records: 1)
static int addr_elem(const bk_ctx* c, const Access& a, uint32_t& el) {
  std::vector<uint64_t> lens;
  if (a.whole) {
    if (c->off) lens.push_back(1);   // record lengths vary: bytes
    else lens.push_back(c->cfg.record_size);
  } else {
    for (uint32_t e = 0; e < a.n_ext; ++e) lens.push_back(a.ext_len[e]);
  }
  auto divides = [&](uint32_t x) {
    for (uint64_t l : lens)
      if (l % x) return false;
    return true;
  };
  el = c->cfg.addr_elem_bytes;
  if (el == 0) {
    el = 8;
    while (el > 1 && !divides(el)) el >>= 1;
    return BK_OK;
  }
  if ((el & (el - 1)) || el > 16 || !divides(el))
    return fail(BK_E_INVAL, "addr_elem_bytes %u must be a power of two <= 16 dividing every accessed length", el);
  return BK_OK;
}

int plan_run_uncached(bk_ctx* c, const Access& a, uint32_t lane_target, Plan& p, uint32_t out_per_rec,
                      int auto_mode, bool user_addr) {
  p.a = a;
  p.user_addr = user_addr;
  if (c->cfg.lane_bytes) lane_target = c->cfg.lane_bytes;
  int mode = (int)c->cfg.gather_mode;
  if (mode == BK_GATHER_FUSED) mode = BK_GATHER_AUTO;   // FUSED is word count's own single-launch path
  if (user_addr) mode = BK_GATHER_ADDR;
  // AUTO (counters in profiles/): whole-record access -> DENSE (copy engine at
  // 55.5 GB/s beats zero-copy's 51.4); sparse access -> HYBRID (host assembly packs exactly the
  // accessed bytes; the zero-copy gather is request-rate bound and only adds capacity on top).
  if (mode == BK_GATHER_AUTO) mode = auto_mode != BK_GATHER_AUTO ? auto_mode : a.whole ? BK_GATHER_DENSE : BK_GATHER_HYBRID;
  if (mode != BK_GATHER_ZC && mode != BK_GATHER_DENSE && mode != BK_GATHER_CPU && mode != BK_GATHER_HYBRID &&
      mode != BK_GATHER_ADDR)
    return fail(BK_E_INVAL, "bad gather_mode %d", mode);
  p.mode = mode;
  if (mode == BK_GATHER_ADDR) {
    const int rc = addr_elem(c, a, p.elem);
    if (rc) return rc;
  }
  p.zero_copy = mode != BK_GATHER_DENSE;
  p.desc_sets = mode == BK_GATHER_ZC ? 2 : 1;
  p.packed = (mode == BK_GATHER_CPU || mode == BK_GATHER_HYBRID) && host_packable(a);
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

int plan_run(bk_ctx* c, const Access& a, uint32_t lane_target, Plan& p, uint32_t out_per_chunk, int auto_mode,
             bool user_addr) {
  char key[256];
  snprintf(key, sizeof key, "%u/%u/%u/%u/%u/%u/%u/%u/%u/%u/%d/%d/%d", a.whole, a.n_ext, a.ext_off[0], a.ext_len[0],
           a.ext_off[1], a.ext_len[1], a.ext_off[2], a.ext_len[2], a.E, lane_target, (int)out_per_chunk, auto_mode,
           (int)user_addr);
  std::string k(key);
  for (uint32_t e = 3; e < a.n_ext; ++e) k += "/" + std::to_string(a.ext_off[e]) + ":" + std::to_string(a.ext_len[e]);
  for (auto& kv : c->plan_cache)
    if (kv.first == k) {
      p = kv.second;
      return BK_OK;
    }
  const int rc = plan_run_uncached(c, a, lane_target, p, out_per_chunk, auto_mode, user_addr);
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
    for (uint32_t d = 0; d < 2; ++d) {
      if (d == 1 && p.desc_sets < 2) {
        s.meta_set[1] = s.meta_set[0];
        s.lanes_set[1] = s.lanes_set[0];
        s.tileK_set[1] = s.tileK_set[0];
        s.tile_base_set[1] = s.tile_base_set[0];
        break;
      }
      s.meta_set[d] = reinterpret_cast<uint64_t*>(q);
      q += align_up(p.meta_cap * 8, kAlign);
      s.lanes_set[d] = reinterpret_cast<LaneDesc*>(q);
      q += align_up((uint64_t)p.L * sizeof(LaneDesc), kAlign);
      s.tileK_set[d] = reinterpret_cast<uint32_t*>(q);
      q += align_up(ntiles * 4, kAlign);
      s.tile_base_set[d] = reinterpret_cast<uint64_t*>(q);
      q += align_up((ntiles + 1) * 8, kAlign);
    }
    s.meta = s.meta_set[0];
    s.lanes = s.lanes_set[0];
    s.tileK = s.tileK_set[0];
    s.tile_base = s.tile_base_set[0];
    s.out = p.out_cap ? q : nullptr;
    q += align_up(p.out_cap, kAlign);
    s.exp = s.uaddr = s.ubase = nullptr;
    s.ecount = s.ucount = nullptr;
    s.epos = nullptr;
    if (p.mode == BK_GATHER_ADDR) {
      s.exp = reinterpret_cast<uint64_t*>(q);
      q += align_up(p.exp_cap, kAlign);
      s.ecount = reinterpret_cast<uint32_t*>(q);
      q += align_up((uint64_t)p.L * 4, kAlign);
      s.epos = reinterpret_cast<uint64_t*>(q);
      q += align_up(((uint64_t)p.L + 1) * 8, kAlign);
      if (p.user_addr) {
        s.uaddr = reinterpret_cast<uint64_t*>(q);
        q += align_up(p.exp_cap, kAlign);
        s.ubase = reinterpret_cast<uint64_t*>(q);
        q += align_up((uint64_t)p.L * 8 + 8, kAlign);
        s.ucount = reinterpret_cast<uint32_t*>(q);
        q += align_up((uint64_t)p.L * 4, kAlign);
      }
    }
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


}  // namespace rt
}  // namespace bk
