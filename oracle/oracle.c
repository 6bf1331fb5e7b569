/* oracle.c — plain single-threaded CPU oracle (TEST INFRASTRUCTURE ONLY; see oracle.h).
 * Built with -O2 -ffp-contract=off (no FMA contraction; fmaf is called explicitly where the
 * definition says so). Written for readability against the paper, not speed. */
#include "oracle.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>

static uint64_t rec_start(const uint64_t* off, uint64_t rec_size, uint64_t r) {
  return off ? off[r] : r * rec_size;
}
static uint64_t rec_end(const uint64_t* off, uint64_t n, uint64_t nbytes, uint64_t rec_size, uint64_t r) {
  if (!off) return (r + 1) * rec_size;
  return r + 1 < n ? off[r + 1] : nbytes;
}

/* ------------------------------------------------------------------ O1 word count */
static int is_delim(uint8_t c) { return c == 0x20 || (c >= 0x09 && c <= 0x0D); }

typedef struct { uint64_t off; uint32_t len; } WordRef;
static const uint8_t* g_text; /* qsort comparator context (single-threaded oracle) */

static int word_cmp(const void* pa, const void* pb) {
  const WordRef* a = (const WordRef*)pa;
  const WordRef* b = (const WordRef*)pb;
  uint32_t m = a->len < b->len ? a->len : b->len;
  int c = memcmp(g_text + a->off, g_text + b->off, m);
  if (c) return c;
  if (a->len != b->len) return a->len < b->len ? -1 : 1;
  return a->off < b->off ? -1 : (a->off > b->off); /* keeps the first occurrence first */
}

int64_t oracle_wc(const uint8_t* text, uint64_t nbytes, const uint64_t* off, uint64_t n,
                  uint64_t* word_off, uint32_t* word_len, uint64_t* word_cnt, uint64_t cap) {
  /* 1. list every word occurrence, record by record */
  uint64_t capw = 1024, nw = 0;
  WordRef* w = (WordRef*)malloc(capw * sizeof(WordRef));
  for (uint64_t r = 0; r < n; ++r) {
    uint64_t s = off[r], e = r + 1 < n ? off[r + 1] : nbytes;
    uint64_t i = s;
    while (i < e) {
      while (i < e && is_delim(text[i])) ++i;
      uint64_t b = i;
      while (i < e && !is_delim(text[i])) ++i;
      if (i > b) {
        if (nw == capw) { capw *= 2; w = (WordRef*)realloc(w, capw * sizeof(WordRef)); }
        w[nw].off = b; w[nw].len = (uint32_t)(i - b); ++nw;
      }
    }
  }
  /* 2. sort occurrences by word bytes, 3. count runs of equal words */
  g_text = text;
  qsort(w, nw, sizeof(WordRef), word_cmp);
  int64_t V = 0;
  for (uint64_t i = 0; i < nw;) {
    uint64_t j = i + 1;
    while (j < nw && w[j].len == w[i].len && memcmp(text + w[j].off, text + w[i].off, w[i].len) == 0) ++j;
    if ((uint64_t)V < cap) { word_off[V] = w[i].off; word_len[V] = w[i].len; word_cnt[V] = j - i; }
    ++V;
    i = j;
  }
  free(w);
  return (uint64_t)V > cap ? -V : V;
}

/* ------------------------------------------------------------------ O2 grep */
int64_t oracle_grep(const uint8_t* d, uint64_t nbytes, const uint64_t* off, uint64_t n,
                    const uint8_t* pat, uint32_t plen, uint64_t first, uint64_t* idx, uint64_t cap) {
  int64_t m = 0;
  for (uint64_t r = 0; r < n; ++r) {
    uint64_t s = off[r], e = r + 1 < n ? off[r + 1] : nbytes;
    if (e - s < 48) return -1;
    const uint8_t* key = d + s + 16;
    uint32_t kl = 0;
    while (kl < 32 && key[kl] != 0) ++kl;
    int hit = 0;
    if (plen == 0) hit = 1;
    for (uint32_t p = 0; !hit && p + plen <= kl; ++p)
      if (memcmp(key + p, pat, plen) == 0) hit = 1;
    if (hit) { if ((uint64_t)m < cap) idx[m] = first + r; ++m; }
  }
  return m;
}

/* ------------------------------------------------------------------ O3 k-means */
static uint64_t mix64(uint64_t x) {
  x ^= x >> 30; x *= 0xbf58476d1ce4e5b9ULL;
  x ^= x >> 27; x *= 0x94d049bb133111ebULL;
  x ^= x >> 31;
  return x;
}

void oracle_kmeans(const float* x, uint64_t n, const float* mu, uint32_t K, uint64_t first,
                   uint64_t* count, double* sum, uint64_t* chk, int32_t* cid) {
  memset(count, 0, sizeof(uint64_t) * K);
  memset(sum, 0, sizeof(double) * K * 16);
  uint64_t c = 0;
  for (uint64_t i = 0; i < n; ++i) {
    const float* p = x + i * 16;
    /* findClosestCluster: argmin over k of the fp32 squared distance, lowest k on ties */
    uint32_t best = 0;
    float bestd = 0.0f;
    for (uint32_t k = 0; k < K; ++k) {
      float acc = 0.0f;
      for (int j = 0; j < 16; ++j) {
        float t = p[j] - mu[k * 16 + j];
        acc = fmaf(t, t, acc);
      }
      if (k == 0 || acc < bestd) { bestd = acc; best = k; }
    }
    count[best] += 1;
    for (int j = 0; j < 16; ++j) sum[best * 16 + j] += (double)p[j];
    c += mix64(((first + i) << 8) ^ (uint64_t)best);
    if (cid) cid[i] = (int32_t)best;
  }
  *chk = c;
}

/* ------------------------------------------------------------------ O4 partition */
int oracle_partition(const uint64_t* kv, uint64_t n, uint32_t B, uint64_t* boff, uint64_t* out) {
  int bits = 0;
  while ((1u << bits) < B) ++bits;
  if ((1u << bits) != B || bits > 16) return -1;
  memset(boff, 0, sizeof(uint64_t) * (B + 1));
  for (uint64_t i = 0; i < n; ++i) {
    uint64_t b = bits ? mix64(kv[2 * i]) >> (64 - bits) : 0;
    boff[b + 1] += 1;
  }
  for (uint32_t b = 0; b < B; ++b) boff[b + 1] += boff[b];
  uint64_t* next = (uint64_t*)malloc(sizeof(uint64_t) * B);
  memcpy(next, boff, sizeof(uint64_t) * B);
  for (uint64_t i = 0; i < n; ++i) {
    uint64_t b = bits ? mix64(kv[2 * i]) >> (64 - bits) : 0;
    uint64_t o = next[b]++;
    out[2 * o] = kv[2 * i];
    out[2 * o + 1] = kv[2 * i + 1];
  }
  free(next);
  return 0;
}

/* ------------------------------------------------------------------ O5 group-by */
int oracle_groupby(const uint8_t* recs, uint64_t n, uint32_t stride, uint32_t G,
                   uint64_t* count, uint64_t* qty, double* amount) {
  memset(count, 0, sizeof(uint64_t) * G);
  memset(qty, 0, sizeof(uint64_t) * G);
  memset(amount, 0, sizeof(double) * G);
  for (uint64_t i = 0; i < n; ++i) {
    uint32_t key, q;
    double a;
    memcpy(&key, recs + i * stride, 4);
    memcpy(&q, recs + i * stride + 4, 4);
    memcpy(&a, recs + i * stride + 8, 8);
    if (key >= G) return -1;
    count[key] += 1;
    qty[key] += q;
    amount[key] += a;
  }
  return 0;
}

/* ------------------------------------------------------------------ O6 k-mers */
static int cmp_u64(const void* a, const void* b) {
  const uint64_t x = *(const uint64_t*)a, y = *(const uint64_t*)b;
  return x < y ? -1 : x > y;
}

int64_t oracle_kmer(const uint8_t* recs, uint64_t n, uint32_t rec_size, uint32_t seq_off, uint32_t seq_len,
                    uint32_t k, uint64_t* kmer, uint64_t* count, uint64_t cap) {
  /* 1. every k-mer occurrence, record by record, window by window */
  uint64_t cap_occ = 1024, m = 0;
  uint64_t* occ = (uint64_t*)malloc(cap_occ * 8);
  for (uint64_t r = 0; r < n; ++r) {
    const uint8_t* s = recs + r * rec_size + seq_off;
    for (uint32_t j = 0; j + k <= seq_len; ++j) {
      uint64_t v = 0;
      int ok = 1;
      for (uint32_t q = 0; q < k && ok; ++q) {
        int code = s[j + q] == 'A' ? 0 : s[j + q] == 'C' ? 1 : s[j + q] == 'G' ? 2 : s[j + q] == 'T' ? 3 : -1;
        if (code < 0) ok = 0;
        else v = v * 4 + (uint64_t)code;
      }
      if (!ok) continue;
      if (m == cap_occ) { cap_occ *= 2; occ = (uint64_t*)realloc(occ, cap_occ * 8); }
      occ[m++] = v;
    }
  }
  /* 2. sort, 3. count runs */
  qsort(occ, m, 8, cmp_u64);
  int64_t V = 0;
  for (uint64_t i = 0; i < m;) {
    uint64_t j = i + 1;
    while (j < m && occ[j] == occ[i]) ++j;
    if ((uint64_t)V < cap) { kmer[V] = occ[i]; count[V] = j - i; }
    ++V;
    i = j;
  }
  free(occ);
  return (uint64_t)V > cap ? -V : V;
}

/* ------------------------------------------------------------------ O-L layout */
/* accessed bytes of record r under the access spec */
static int64_t rec_access(const uint64_t* off, uint64_t n, uint64_t nbytes, uint64_t rec_size,
                          uint32_t n_ext, const uint32_t* ext_off, const uint32_t* ext_len, uint64_t r) {
  uint64_t len = rec_end(off, n, nbytes, rec_size, r) - rec_start(off, rec_size, r);
  if (n_ext == 0) return (int64_t)len;
  int64_t a = 0;
  for (uint32_t e = 0; e < n_ext; ++e) {
    if ((uint64_t)ext_off[e] + ext_len[e] > len) return -1;
    a += ext_len[e];
  }
  return a;
}

int64_t oracle_plan_chunks(const uint64_t* off, uint64_t n, uint64_t nbytes, uint64_t rec_size,
                           uint32_t n_ext, const uint32_t* ext_off, const uint32_t* ext_len,
                           uint64_t budget, uint64_t* bounds, uint64_t cap) {
  int64_t C = 0;
  uint64_t lo = 0;
  if (cap < 1) return -2;
  bounds[0] = 0;
  while (lo < n) {
    uint64_t acc = 0, r = lo;
    while (r < n) {
      int64_t a = rec_access(off, n, nbytes, rec_size, n_ext, ext_off, ext_len, r);
      if (a < 0) return -1;
      if (acc + (uint64_t)a > budget) break;
      acc += (uint64_t)a;
      ++r;
    }
    if (r == lo) return -1; /* one record exceeds the budget: BK_E_RANGE */
    ++C;
    if ((uint64_t)C >= cap) return -2;
    bounds[C] = r;
    lo = r;
  }
  return C;
}

int64_t oracle_layout(const uint8_t* d, const uint64_t* off, uint64_t n, uint64_t nbytes,
                      uint64_t rec_size, uint32_t n_ext, const uint32_t* ext_off, const uint32_t* ext_len,
                      uint64_t lo, uint64_t hi, uint32_t L,
                      uint64_t* lane_first, uint64_t* lane_nrec, uint64_t* lane_bytes,
                      uint8_t* stage, uint64_t cap) {
  if (L == 0 || L % 32 || lo > hi || hi > n) return -1;
  /* prefix A(lo, r) for r in [lo, hi] */
  uint64_t m = hi - lo;
  uint64_t* A = (uint64_t*)malloc(sizeof(uint64_t) * (m + 1));
  A[0] = 0;
  for (uint64_t r = lo; r < hi; ++r) {
    int64_t a = rec_access(off, n, nbytes, rec_size, n_ext, ext_off, ext_len, r);
    if (a < 0) { free(A); return -1; }
    A[r - lo + 1] = A[r - lo] + (uint64_t)a;
  }
  uint64_t total = A[m];
  /* lane boundaries: first(t) = min r with A(lo,r) >= floor(t*total/L) */
  uint64_t* first = (uint64_t*)malloc(sizeof(uint64_t) * (L + 1));
  for (uint32_t t = 0; t < L; ++t) {
    uint64_t target = (uint64_t)(((unsigned __int128)t * total) / L);
    uint64_t r = 0;
    while (A[r] < target) ++r;
    first[t] = lo + r;
  }
  first[L] = hi;
  /* warp tiles */
  uint64_t size = 0;
  uint64_t* tile_base = (uint64_t*)malloc(sizeof(uint64_t) * (L / 32));
  for (uint32_t w = 0; w < L / 32; ++w) {
    uint64_t K = 0;
    for (uint32_t t = 32 * w; t < 32 * w + 32; ++t) {
      uint64_t bytes = A[first[t + 1] - lo] - A[first[t] - lo];
      uint64_t W = (bytes + 15) / 16;
      if (W > K) K = W;
      lane_first[t] = first[t];
      lane_nrec[t] = first[t + 1] - first[t];
      lane_bytes[t] = bytes;
    }
    tile_base[w] = size;
    size += 512 * K;
  }
  if (stage) {
    if (size > cap) { free(A); free(first); free(tile_base); return -1; }
    memset(stage, 0, size);
    for (uint32_t t = 0; t < L; ++t) {
      uint64_t b = 0; /* byte index within S_t */
      for (uint64_t r = first[t]; r < first[t + 1]; ++r) {
        uint64_t s = rec_start(off, rec_size, r);
        uint64_t e = rec_end(off, n, nbytes, rec_size, r);
        uint32_t ne = n_ext ? n_ext : 1;
        for (uint32_t x = 0; x < ne; ++x) {
          uint64_t xs = n_ext ? s + ext_off[x] : s;
          uint64_t xl = n_ext ? ext_len[x] : e - s;
          for (uint64_t q = 0; q < xl; ++q, ++b) {
            uint64_t k = b / 16;
            stage[tile_base[t / 32] + (k * 32 + t % 32) * 16 + b % 16] = d[xs + q];
          }
        }
      }
    }
  }
  free(A); free(first); free(tile_base);
  return (int64_t)size;
}

/* ------------------------------------------------------------------ O-P pattern */
int oracle_pattern_online(const uint64_t* a, uint64_t n, uint32_t T, uint32_t pmax, int64_t* strides) {
  uint32_t first = n < T ? (uint32_t)n : T;
  int p = oracle_pattern(a, first, pmax, strides);
  if (p == 0) return 0;
  for (uint64_t k = first; k < n; ++k)   /* verify each subsequently generated address */
    if ((int64_t)(a[k] - a[k - 1]) != strides[(k - 1) % (uint64_t)p]) return 0;
  return p;
}

int oracle_pattern(const uint64_t* a, uint32_t n, uint32_t pmax, int64_t* strides) {
  if (n < 2) return 0;
  for (uint32_t p = 1; p <= pmax && p + 1 < n; ++p) { /* >= 1 delta beyond the first period verifies it */
    int ok = 1;
    for (uint32_t k = 0; k + 1 < n && ok; ++k)
      if ((int64_t)(a[k + 1] - a[k]) != (int64_t)(a[(k % p) + 1] - a[k % p])) ok = 0;
    if (ok) {
      for (uint32_t q = 0; q < p; ++q) strides[q] = (int64_t)(a[q + 1] - a[q]);
      return (int)p;
    }
  }
  return 0;
}
