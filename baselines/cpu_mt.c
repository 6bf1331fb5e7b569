/* cpu_mt.c — the paper's multithreaded CPU variant (ii), the comparison
 * point of its "3.0x over multithreaded CPU" claim. Bench-only baseline: OpenMP over all
 * host cores, each thread a contiguous record range, per-thread partial results merged at the end.
 * Not the oracle (oracle/ stays single-threaded and unoptimised) and not part of libbk. */
#include <math.h>
#include <omp.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

int mt_threads(void) { return omp_get_max_threads(); }

/* grep: returns the match count; indices are written in ascending order (per-thread buffers). */
int64_t mt_grep(const uint8_t* d, uint64_t nbytes, const uint64_t* off, uint64_t n, const uint8_t* pat,
                uint32_t plen, uint64_t* idx, uint64_t cap) {
  int T = omp_get_max_threads();
  uint64_t* cnt = calloc(T + 1, sizeof(uint64_t));
  uint64_t** loc = calloc(T, sizeof(uint64_t*));
#pragma omp parallel num_threads(T)
  {
    int t = omp_get_thread_num();
    uint64_t lo = n * t / T, hi = n * (t + 1) / T, m = 0, capl = 1024;
    uint64_t* buf = malloc(capl * 8);
    for (uint64_t r = lo; r < hi; ++r) {
      const uint8_t* key = d + off[r] + 16;
      uint32_t kl = 0;
      while (kl < 32 && key[kl]) ++kl;
      int hit = plen == 0;
      for (uint32_t p = 0; !hit && p + plen <= kl; ++p) hit = memcmp(key + p, pat, plen) == 0;
      if (hit) {
        if (m == capl) { capl *= 2; buf = realloc(buf, capl * 8); }
        buf[m++] = r;
      }
    }
    loc[t] = buf;
    cnt[t + 1] = m;
  }
  for (int t = 0; t < T; ++t) cnt[t + 1] += cnt[t];
#pragma omp parallel for num_threads(T)
  for (int t = 0; t < T; ++t) {
    for (uint64_t i = cnt[t]; i < cnt[t + 1] && i < cap; ++i) idx[i] = loc[t][i - cnt[t]];
    free(loc[t]);
  }
  int64_t total = (int64_t)cnt[T];
  free(cnt);
  free(loc);
  (void)nbytes;
  return total;
}

void mt_groupby(const uint8_t* recs, uint64_t n, uint32_t stride, uint32_t G, uint64_t* count, uint64_t* qty,
                double* amount) {
  memset(count, 0, 8 * G);
  memset(qty, 0, 8 * G);
  memset(amount, 0, 8 * G);
#pragma omp parallel
  {
    uint64_t* c = calloc(G, 8);
    uint64_t* q = calloc(G, 8);
    double* a = calloc(G, 8);
#pragma omp for schedule(static)
    for (uint64_t i = 0; i < n; ++i) {
      uint32_t k, qq;
      double aa;
      memcpy(&k, recs + i * stride, 4);
      memcpy(&qq, recs + i * stride + 4, 4);
      memcpy(&aa, recs + i * stride + 8, 8);
      if (k < G) { c[k] += 1; q[k] += qq; a[k] += aa; }
    }
#pragma omp critical
    for (uint32_t g = 0; g < G; ++g) { count[g] += c[g]; qty[g] += q[g]; amount[g] += a[g]; }
    free(c);
    free(q);
    free(a);
  }
}

void mt_kmeans(const float* x, uint64_t n, const float* mu, uint32_t K, uint64_t* count, double* sum) {
  memset(count, 0, 8 * K);
  memset(sum, 0, 8 * K * 16);
#pragma omp parallel
  {
    uint64_t* c = calloc(K, 8);
    double* s = calloc((size_t)K * 16, 8);
#pragma omp for schedule(static)
    for (uint64_t i = 0; i < n; ++i) {
      const float* p = x + i * 16;
      uint32_t best = 0;
      float bd = 0;
      for (uint32_t k = 0; k < K; ++k) {
        float acc = 0;
        for (int j = 0; j < 16; ++j) { float t = p[j] - mu[k * 16 + j]; acc = fmaf(t, t, acc); }
        if (k == 0 || acc < bd) { bd = acc; best = k; }
      }
      c[best] += 1;
      for (int j = 0; j < 16; ++j) s[best * 16 + j] += p[j];
    }
#pragma omp critical
    for (uint32_t k = 0; k < K * 16; ++k) { sum[k] += s[k]; if (k < K) count[k] += c[k]; }
    free(c);
    free(s);
  }
}

/* ---- partition (C4): stable bucket-major partition by mix64(key) >> (64 - log2 B) ----------------
 * Two passes over per-thread contiguous ranges: per-thread bucket histograms, a (bucket, thread)
 * exclusive scan, then a stable scatter. boff: B+1 bucket offsets. */
static inline uint64_t mt_mix64(uint64_t x) {
  x ^= x >> 30; x *= 0xbf58476d1ce4e5b9ull;
  x ^= x >> 27; x *= 0x94d049bb133111ebull;
  x ^= x >> 31;
  return x;
}

void mt_partition(const uint64_t* kv, uint64_t n, uint32_t B, uint64_t* out, uint64_t* boff) {
  int bits = 0;
  while ((1u << bits) < B) ++bits;
  const int T = omp_get_max_threads();
  uint64_t* h = calloc((size_t)T * B, 8);
#pragma omp parallel num_threads(T)
  {
    const int t = omp_get_thread_num();
    const uint64_t lo = n * t / T, hi = n * (t + 1) / T;
    uint64_t* ht = h + (size_t)t * B;
    for (uint64_t i = lo; i < hi; ++i) ht[bits ? mt_mix64(kv[2 * i]) >> (64 - bits) : 0]++;
#pragma omp barrier
#pragma omp single
    {
      uint64_t acc = 0;
      for (uint32_t b = 0; b < B; ++b) {
        boff[b] = acc;
        for (int u = 0; u < T; ++u) { const uint64_t c = h[(size_t)u * B + b]; h[(size_t)u * B + b] = acc; acc += c; }
      }
      boff[B] = acc;
    }
    for (uint64_t i = lo; i < hi; ++i) {
      const uint64_t b = bits ? mt_mix64(kv[2 * i]) >> (64 - bits) : 0;
      const uint64_t p = ht[b]++;
      out[2 * p] = kv[2 * i];
      out[2 * p + 1] = kv[2 * i + 1];
    }
  }
  free(h);
}

/* ---- k-mers (f4): exact-key concurrent open-addressing table (key = 2-bit k-mer + 1) ------------
 * Returns the number of distinct k-mers written (unordered) to kmer/cnt, or -(needed) if cap is
 * too small; -1 if the table filled up. */
int64_t mt_kmer(const uint8_t* recs, uint64_t n, uint32_t rec_size, uint32_t seq_off, uint32_t seq_len, uint32_t k,
                uint64_t slots, uint64_t* kmer, uint64_t* cnt, uint64_t cap) {
  uint64_t* key = calloc(slots, 8);
  uint64_t* val = calloc(slots, 8);
  const uint64_t mask = slots - 1, kmask = k == 32 ? ~0ull : ((1ull << (2 * k)) - 1);
  int full = 0;
#pragma omp parallel for schedule(dynamic, 4096) reduction(| : full)
  for (uint64_t r = 0; r < n; ++r) {
    const uint8_t* s = recs + r * rec_size + seq_off;
    uint64_t v = 0;
    uint32_t valid = 0;
    for (uint32_t i = 0; i < seq_len; ++i) {
      const uint8_t ch = s[i];
      const int code = ch == 'A' ? 0 : ch == 'C' ? 1 : ch == 'G' ? 2 : ch == 'T' ? 3 : -1;
      if (code < 0) { valid = 0; v = 0; continue; }
      v = ((v << 2) | (uint64_t)code) & kmask;
      if (++valid < k) continue;
      const uint64_t kk = v + 1;
      uint64_t slot = mt_mix64(kk) & mask, probe = 0;
      for (; probe <= mask; ++probe, slot = (slot + 1) & mask) {
        uint64_t cur = __atomic_load_n(&key[slot], __ATOMIC_RELAXED);
        if (cur == 0) {
          uint64_t z = 0;
          if (__atomic_compare_exchange_n(&key[slot], &z, kk, 0, __ATOMIC_RELAXED, __ATOMIC_RELAXED)) cur = kk;
          else cur = z;
        }
        if (cur == kk) { __atomic_fetch_add(&val[slot], 1, __ATOMIC_RELAXED); break; }
      }
      if (probe > mask) full = 1;
    }
  }
  int64_t V = 0;
  if (!full) {
    for (uint64_t i = 0; i < slots; ++i)
      if (key[i]) {
        if ((uint64_t)V < cap) { kmer[V] = key[i] - 1; cnt[V] = val[i]; }
        ++V;
      }
    if ((uint64_t)V > cap) V = -V;
  }
  free(key);
  free(val);
  return full ? -1 : V;
}

/* ---- word count (C1): per-thread exact tables (FNV-1a hash + byte compare), merged at the end ----
 * Word = maximal run of bytes outside {0x20, 0x09..0x0D} inside one record (A10/A19).
 * Output: unordered (offset of one occurrence, length, count); returns the number of distinct words,
 * or -(needed) if cap is too small. */
typedef struct { uint64_t h, off, len, cnt; } mt_wc_e;
typedef struct { mt_wc_e* e; uint64_t mask, used; } mt_wc_t;

static int mt_isdelim(uint8_t c) { return c == 0x20 || (uint8_t)(c - 0x09) <= 4; }

static void mt_wc_init(mt_wc_t* t, uint64_t slots) {
  t->e = calloc(slots, sizeof(mt_wc_e));
  t->mask = slots - 1;
  t->used = 0;
}

static void mt_wc_add(mt_wc_t* t, const uint8_t* d, uint64_t h, uint64_t off, uint64_t len, uint64_t cnt);

static void mt_wc_grow(mt_wc_t* t, const uint8_t* d) {
  mt_wc_t n;
  mt_wc_init(&n, (t->mask + 1) * 2);
  for (uint64_t i = 0; i <= t->mask; ++i)
    if (t->e[i].cnt) mt_wc_add(&n, d, t->e[i].h, t->e[i].off, t->e[i].len, t->e[i].cnt);
  free(t->e);
  *t = n;
}

static void mt_wc_add(mt_wc_t* t, const uint8_t* d, uint64_t h, uint64_t off, uint64_t len, uint64_t cnt) {
  if ((t->used + 1) * 10 > (t->mask + 1) * 7) mt_wc_grow(t, d);
  for (uint64_t s = h & t->mask;; s = (s + 1) & t->mask) {
    mt_wc_e* e = &t->e[s];
    if (!e->cnt) { e->h = h; e->off = off; e->len = len; e->cnt = cnt; t->used++; return; }
    if (e->h == h && e->len == len && memcmp(d + e->off, d + off, len) == 0) { e->cnt += cnt; return; }
  }
}

int64_t mt_wordcount(const uint8_t* d, uint64_t nbytes, const uint64_t* off, uint64_t n, uint64_t* w_off,
                     uint32_t* w_len, uint64_t* w_cnt, uint64_t cap) {
  const int T = omp_get_max_threads();
  mt_wc_t* tabs = calloc(T, sizeof(mt_wc_t));
#pragma omp parallel num_threads(T)
  {
    const int t = omp_get_thread_num();
    const uint64_t lo = n * t / T, hi = n * (t + 1) / T;
    mt_wc_init(&tabs[t], 1u << 16);
    for (uint64_t r = lo; r < hi; ++r) {
      const uint64_t a = off[r], b = r + 1 < n ? off[r + 1] : nbytes;
      uint64_t i = a;
      while (i < b) {
        while (i < b && mt_isdelim(d[i])) ++i;
        const uint64_t s = i;
        uint64_t h = 0xcbf29ce484222325ull;
        while (i < b && !mt_isdelim(d[i])) { h = (h ^ d[i]) * 0x100000001b3ull; ++i; }
        if (i > s) mt_wc_add(&tabs[t], d, mt_mix64(h ^ (i - s)), s, i - s, 1);
      }
    }
  }
  mt_wc_t g;
  mt_wc_init(&g, 1u << 17);
  for (int t = 0; t < T; ++t) {
    for (uint64_t i = 0; i <= tabs[t].mask; ++i)
      if (tabs[t].e[i].cnt) mt_wc_add(&g, d, tabs[t].e[i].h, tabs[t].e[i].off, tabs[t].e[i].len, tabs[t].e[i].cnt);
    free(tabs[t].e);
  }
  free(tabs);
  int64_t V = 0;
  for (uint64_t i = 0; i <= g.mask; ++i)
    if (g.e[i].cnt) {
      if ((uint64_t)V < cap) { w_off[V] = g.e[i].off; w_len[V] = (uint32_t)g.e[i].len; w_cnt[V] = g.e[i].cnt; }
      ++V;
    }
  free(g.e);
  return (uint64_t)V > cap ? -V : V;
}
