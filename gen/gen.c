/* gen.c — seeded synthetic input generators. See gen.h; recipes in DESIGN.md §Inputs.
 * Input generation only: nothing here is part of either computation. */
#include "gen.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>
#include <sys/mman.h>

static inline uint64_t mix64(uint64_t x) {
  x ^= x >> 30; x *= 0xbf58476d1ce4e5b9ULL;
  x ^= x >> 27; x *= 0x94d049bb133111ebULL;
  x ^= x >> 31;
  return x;
}

uint64_t gen_R(uint64_t seed, uint64_t stream, uint64_t i) {
  return mix64(mix64(seed ^ (stream * 0xD1B54A32D192ED03ULL)) + i * 0x9E3779B97F4A7C15ULL);
}

/* U in [0,1) with 24 random bits. */
static inline double gen_U(uint64_t seed, uint64_t stream, uint64_t i) {
  return (double)(gen_R(seed, stream, i) >> 40) * (1.0 / 16777216.0);
}

/* Zipf(1.0) over [0, V): inverse CDF by binary search on a cumulative table. */
static double* zipf_cdf(uint32_t V) {
  double* cdf = (double*)malloc(sizeof(double) * V);
  double s = 0;
  for (uint32_t v = 0; v < V; ++v) { s += 1.0 / (double)(v + 1); cdf[v] = s; }
  for (uint32_t v = 0; v < V; ++v) cdf[v] /= s;
  return cdf;
}
static uint32_t zipf_pick(const double* cdf, uint32_t V, double u) {
  uint32_t lo = 0, hi = V - 1;
  while (lo < hi) { uint32_t mid = (lo + hi) / 2; if (cdf[mid] > u) hi = mid; else lo = mid + 1; }
  return lo;
}

/* ---------------- C1: text ---------------- */
#define WC_VOCAB 65536u
int gen_text(uint64_t seed, uint64_t cap_bytes, uint8_t* buf, uint64_t* off, uint64_t cap_recs,
             uint64_t* out_nbytes, uint64_t* out_nrec) {
  double* cdf = zipf_cdf(WC_VOCAB);
  /* spelling of vocabulary word v: length 1 + R%12, lowercase letters */
  uint8_t* spell = (uint8_t*)malloc((size_t)WC_VOCAB * 12);
  uint8_t* slen = (uint8_t*)malloc(WC_VOCAB);
  if (!cdf || !spell || !slen) { free(cdf); free(spell); free(slen); return -1; }
  for (uint32_t v = 0; v < WC_VOCAB; ++v) {
    slen[v] = (uint8_t)(1 + gen_R(seed, 10, v) % 12);
    for (int j = 0; j < slen[v]; ++j) spell[(size_t)v * 12 + j] = (uint8_t)('a' + gen_R(seed, 11, (uint64_t)v * 16 + j) % 26);
  }
  uint64_t pos = 0, line = 0;
  uint8_t tmp[16 * 13 + 1];
  for (;;) {
    if (line >= cap_recs) break;
    uint32_t nw = (uint32_t)(gen_R(seed, 1, line) % 17);
    size_t L = 0;
    for (uint32_t j = 0; j < nw; ++j) {
      uint32_t v = zipf_pick(cdf, WC_VOCAB, gen_U(seed, 2, line * 16 + j));
      if (j) tmp[L++] = ' ';
      memcpy(tmp + L, spell + (size_t)v * 12, slen[v]);
      L += slen[v];
    }
    tmp[L++] = '\n';
    if (pos + L > cap_bytes) break;
    off[line] = pos;
    memcpy(buf + pos, tmp, L);
    pos += L;
    ++line;
  }
  free(cdf); free(spell); free(slen);
  *out_nbytes = pos;
  *out_nrec = line;
  return 0;
}

/* ---------------- C2: grep records ---------------- */
static inline uint64_t grep_len(uint64_t seed, uint64_t i) { return 48 + 8 * (gen_R(seed, 1, i) % 53); }

uint64_t gen_grep_sizes(uint64_t seed, uint64_t first, uint64_t n, uint64_t* off) {
  uint64_t pos = 0;
  for (uint64_t k = 0; k < n; ++k) { off[k] = pos; pos += grep_len(seed, first + k); }
  return pos;
}

uint64_t gen_grep_count_for_bytes(uint64_t seed, uint64_t first, uint64_t max_bytes) {
  uint64_t pos = 0, k = 0;
  for (;; ++k) {
    uint64_t L = grep_len(seed, first + k);
    if (pos + L > max_bytes) break;
    pos += L;
  }
  return k;
}

void gen_grep_fill(uint64_t seed, uint64_t first, uint64_t n, const uint64_t* off, uint8_t* buf, int threads) {
  (void)threads;
#pragma omp parallel for schedule(dynamic, 4096) num_threads(threads > 0 ? threads : 1)
  for (uint64_t k = 0; k < n; ++k) {
    uint64_t i = first + k;
    uint8_t* r = buf + off[k];
    uint32_t len = (uint32_t)grep_len(seed, i);
    uint32_t flags = (uint32_t)(gen_R(seed, 6, i) & 0xffffffffu);
    memcpy(r, &len, 4);
    memcpy(r + 4, &flags, 4);
    memcpy(r + 8, &i, 8);
    uint8_t* key = r + 16;
    memset(key, 0, 32);
    uint32_t kl = (uint32_t)(8 + gen_R(seed, 2, i) % 25); /* 8..32 */
    uint64_t bits = 0;
    for (uint32_t j = 0; j < kl; ++j) {
      if ((j & 7) == 0) bits = gen_R(seed, 3, i * 4 + j / 8);
      key[j] = (uint8_t)('a' + (bits & 0xff) % 26);
      bits >>= 8;
    }
    if (gen_R(seed, 4, i) % 100 == 0) {
      uint32_t p = (uint32_t)(gen_R(seed, 5, i) % (kl - 3));
      memcpy(key + p, "bigk", 4);
    }
    /* printable payload, 8 bytes per draw */
    uint8_t* pay = r + 48;
    uint32_t plen = len - 48;
    for (uint32_t j = 0; j < plen; j += 8) {
      uint64_t b = gen_R(seed, 7, i * 64 + j / 8);
      for (uint32_t q = 0; q < 8 && j + q < plen; ++q) { pay[j + q] = (uint8_t)(0x20 + (b & 0xff) % 95); b >>= 8; }
    }
  }
}

/* ---------------- C3: points ---------------- */
void gen_points(uint64_t seed, uint64_t first, uint64_t n, float* x, int threads) {
  double centre[64][16];
  for (int b = 0; b < 64; ++b)
    for (int j = 0; j < 16; ++j) centre[b][j] = 20.0 + 60.0 * gen_U(seed, 100, (uint64_t)b * 16 + j);
  const double s3 = sqrt(3.0);
#pragma omp parallel for schedule(static) num_threads(threads > 0 ? threads : 1)
  for (uint64_t k = 0; k < n; ++k) {
    uint64_t i = first + k;
    int b = (int)(gen_R(seed, 1, i) % 64);
    for (int j = 0; j < 16; ++j) {
      uint64_t c = i * 16 + j;
      double ih = gen_U(seed, 2, c) + gen_U(seed, 3, c) + gen_U(seed, 4, c) + gen_U(seed, 5, c) - 2.0;
      x[k * 16 + j] = (float)(centre[b][j] + 4.0 * s3 * ih);
    }
  }
}

/* ---------------- C4: key/value ---------------- */
void gen_kv(uint64_t seed, uint64_t first, uint64_t n, uint64_t* kv, int threads) {
#pragma omp parallel for schedule(static) num_threads(threads > 0 ? threads : 1)
  for (uint64_t k = 0; k < n; ++k) {
    uint64_t i = first + k;
    kv[2 * k] = gen_R(seed, 1, i);
    kv[2 * k + 1] = i;
  }
}

/* ---------------- C5: group-by ---------------- */
void gen_groupby(uint64_t seed, uint64_t first, uint64_t n, uint32_t G, uint32_t stride, int zipf,
                 uint8_t* buf, int threads) {
  double* cdf = zipf ? zipf_cdf(G) : NULL;
#pragma omp parallel for schedule(static) num_threads(threads > 0 ? threads : 1)
  for (uint64_t k = 0; k < n; ++k) {
    uint64_t i = first + k;
    uint8_t* r = buf + k * stride;
    uint32_t key = zipf ? zipf_pick(cdf, G, gen_U(seed, 1, i)) : (uint32_t)(gen_R(seed, 1, i) % G);
    uint32_t qty = (uint32_t)(1 + gen_R(seed, 2, i) % 100);
    double amount = (double)(gen_R(seed, 3, i) % 100000) / 100.0;
    memcpy(r, &key, 4);
    memcpy(r + 4, &qty, 4);
    memcpy(r + 8, &amount, 8);
    for (uint32_t j = 16; j < stride; j += 8) {
      uint64_t f = gen_R(seed, 4, i * 8 + j / 8);
      memcpy(r + j, &f, stride - j >= 8 ? 8 : stride - j);
    }
  }
  free(cdf);
}

/* ---------------- host buffers (2 MiB aligned, optionally transparent huge pages) ---------------- */
void* gen_alloc(uint64_t bytes, int huge, void** base_out, uint64_t* len_out) {
  const uint64_t A = 2ull << 20;
  uint64_t len = bytes + A;
  void* base = mmap(NULL, len, PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
  if (base == MAP_FAILED) return NULL;
  uint8_t* p = (uint8_t*)(((uintptr_t)base + A - 1) & ~(uintptr_t)(A - 1));
  if (huge) madvise(p, (bytes + A - 1) & ~(A - 1), MADV_HUGEPAGE);
  *base_out = base;
  *len_out = len;
  return p;
}

void gen_free(void* base, uint64_t len) { munmap(base, len); }

/* ---------------- f4: DNA reads (Table I DNA assembly: fixed-length fragments, 36% read) ----------------
 * Record (256 B): [u64 id][u32 genome_pos][u32 flags][char seq[96] ACGT/N][char qual[144]].
 * A seeded random genome of genome_len bases; read i = the 96 bases at a random position with
 * substitution errors (err_pm per mille) and 'N' calls (n_pm per mille). */
static inline uint8_t genome_base(uint64_t seed, uint64_t p) {
  return (uint8_t)("ACGT"[(gen_R(seed, 20, p >> 5) >> (2 * (p & 31))) & 3]);
}

void gen_dna(uint64_t seed, uint64_t first, uint64_t n, uint64_t genome_len, uint32_t err_pm, uint32_t n_pm,
             uint8_t* buf, int threads) {
#pragma omp parallel for schedule(static) num_threads(threads > 0 ? threads : 1)
  for (uint64_t k = 0; k < n; ++k) {
    const uint64_t i = first + k;
    uint8_t* r = buf + k * 256;
    const uint64_t pos = gen_R(seed, 21, i) % (genome_len - 96);
    const uint32_t pos32 = (uint32_t)pos, flags = 0;
    memcpy(r, &i, 8);
    memcpy(r + 8, &pos32, 4);
    memcpy(r + 12, &flags, 4);
    for (int j = 0; j < 96; ++j) {
      uint8_t b = genome_base(seed, pos + j);
      const uint64_t e = gen_R(seed, 22, i * 96 + j) % 1000;
      if (e < n_pm) b = 'N';
      else if (e < n_pm + err_pm) b = (uint8_t)("ACGT"[gen_R(seed, 23, i * 96 + j) & 3]);
      r[16 + j] = b;
    }
    for (int j = 112; j < 256; j += 8) {
      uint64_t q = gen_R(seed, 24, i * 32 + j / 8);
      for (int t = 0; t < 8; ++t) { r[j + t] = (uint8_t)(33 + (q & 0xff) % 42); q >>= 8; }
    }
  }
}
