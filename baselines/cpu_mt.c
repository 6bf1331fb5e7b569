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
void mt_set_threads(int n) { if (n > 0) omp_set_num_threads(n); }

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

/* ---- word count (C1): per-thread tables merged by hash shard -----------------------------------
 * Word = maximal run of bytes outside {0x20, 0x09..0x0D} inside one record (A10/A19).
 * Word identity = (two independent 64-bit hashes, length), the same reading the GPU path uses
 * (DESIGN.md §2): 32-B entries, no second look at the text. Output: unordered (offset of one
 * occurrence, length, count); returns the number of distinct words, or -(needed) if cap is too small. */
typedef struct { uint64_t h1, h2l, off, cnt; } mt_wc_e;   /* h2l = (h2 << 24) | len */
typedef struct { mt_wc_e* e; uint64_t mask, used; } mt_wc_t;

static int mt_isdelim(uint8_t c) { return c == 0x20 || (uint8_t)(c - 0x09) <= 4; }

static void mt_wc_init(mt_wc_t* t, uint64_t slots) {
  t->e = calloc(slots, sizeof(mt_wc_e));
  t->mask = slots - 1;
  t->used = 0;
}

static void mt_wc_put(mt_wc_t* t, const mt_wc_e* x);

static void mt_wc_grow(mt_wc_t* t) {
  mt_wc_t n;
  mt_wc_init(&n, (t->mask + 1) * 2);
  for (uint64_t i = 0; i <= t->mask; ++i)
    if (t->e[i].cnt) mt_wc_put(&n, &t->e[i]);
  free(t->e);
  *t = n;
}

static void mt_wc_put(mt_wc_t* t, const mt_wc_e* x) {
  if ((t->used + 1) * 10 > (t->mask + 1) * 7) mt_wc_grow(t);
  for (uint64_t s = x->h1 & t->mask;; s = (s + 1) & t->mask) {
    mt_wc_e* e = &t->e[s];
    if (!e->cnt) { *e = *x; t->used++; return; }
    if (e->h1 == x->h1 && e->h2l == x->h2l) { e->cnt += x->cnt; return; }
  }
}

int64_t mt_wordcount(const uint8_t* d, uint64_t nbytes, const uint64_t* off, uint64_t n, uint64_t* w_off,
                     uint32_t* w_len, uint64_t* w_cnt, uint64_t cap) {
  const int T = omp_get_max_threads();
  mt_wc_t* loc = calloc(T, sizeof(mt_wc_t));
  mt_wc_t* shard = calloc(T, sizeof(mt_wc_t));
  uint64_t* base = calloc(T + 1, 8);
  mt_wc_e*** parts = calloc(T, sizeof(mt_wc_e**));
  uint64_t** pcnt = calloc(T, sizeof(uint64_t*));
#pragma omp parallel num_threads(T)
  {
    const int t = omp_get_thread_num();
    const uint64_t lo = n * t / T, hi = n * (t + 1) / T;
    /* the per-thread table is kept across calls (steady state: no page faults / munmap shootdowns
       in the timed region, which otherwise serialise 16 threads on the address-space lock) */
    static mt_wc_e* keep[256];
    static uint64_t keep_slots[256];
    const uint64_t want = 1u << 17;
    if (t < 256 && keep_slots[t] >= want) {
      memset(keep[t], 0, keep_slots[t] * sizeof(mt_wc_e));
      loc[t].e = keep[t];
      loc[t].mask = keep_slots[t] - 1;
      loc[t].used = 0;
    } else {
      mt_wc_init(&loc[t], want);
    }
    mt_wc_e x;
    x.cnt = 1;
    for (uint64_t r = lo; r < hi; ++r) {
      const uint64_t a = off[r], b = r + 1 < n ? off[r + 1] : nbytes;
      uint64_t i = a;
      while (i < b) {
        while (i < b && mt_isdelim(d[i])) ++i;
        const uint64_t s0 = i;
        uint64_t h1 = 0xcbf29ce484222325ull, h2 = 0x84222325cbf29ce4ull;
        while (i < b && !mt_isdelim(d[i])) {
          h1 = (h1 ^ d[i]) * 0x100000001b3ull;
          h2 = (h2 + d[i] + 1) * 0x9E3779B97F4A7C15ull;
          ++i;
        }
        if (i == s0) continue;
        x.h1 = mt_mix64(h1 ^ (i - s0));
        x.h2l = (mt_mix64(h2 + (i - s0)) << 24) | (i - s0);
        x.off = s0;
        mt_wc_put(&loc[t], &x);
      }
    }
    /* split this thread's table by shard (one pass over its own entries) */
    uint64_t* nb = calloc(T, 8);
    for (uint64_t i = 0; i <= loc[t].mask; ++i)
      if (loc[t].e[i].cnt) nb[(loc[t].e[i].h1 >> 40) % (uint64_t)T]++;
    mt_wc_e** lst = calloc(T, sizeof(mt_wc_e*));
    for (int u = 0; u < T; ++u) lst[u] = malloc((nb[u] + 1) * sizeof(mt_wc_e));
    uint64_t* k = calloc(T, 8);
    for (uint64_t i = 0; i <= loc[t].mask; ++i)
      if (loc[t].e[i].cnt) {
        const int u = (int)((loc[t].e[i].h1 >> 40) % (uint64_t)T);
        lst[u][k[u]++] = loc[t].e[i];
      }
    parts[t] = lst;
    pcnt[t] = nb;
    free(k);
#pragma omp barrier
    /* merge: thread t owns the words of shard t, from every thread's list t */
    mt_wc_init(&shard[t], 1u << 14);
    for (int u = 0; u < T; ++u)
      for (uint64_t i = 0; i < pcnt[u][t]; ++i) mt_wc_put(&shard[t], &parts[u][t][i]);
#pragma omp barrier
    for (int u = 0; u < T; ++u) free(lst[u]);
    free(lst);
    free(nb);
    if (t < 256) {   /* keep this thread's table for the next call */
      keep[t] = loc[t].e;   /* mt_wc_grow already freed the previous one if the table grew */
      keep_slots[t] = loc[t].mask + 1;
    } else {
      free(loc[t].e);
    }
    base[t + 1] = shard[t].used;
#pragma omp barrier
#pragma omp single
    for (int u = 0; u < T; ++u) base[u + 1] += base[u];
    uint64_t v = base[t];
    for (uint64_t i = 0; i <= shard[t].mask; ++i) {
      const mt_wc_e* e = &shard[t].e[i];
      if (!e->cnt) continue;
      if (v < cap) { w_off[v] = e->off; w_len[v] = (uint32_t)(e->h2l & 0xffffff); w_cnt[v] = e->cnt; }
      ++v;
    }
    free(shard[t].e);
  }
  const int64_t V = (int64_t)base[T];
  free(loc);
  free(shard);
  free(base);
  free(parts);
  free(pcnt);
  return (uint64_t)V > cap ? -V : V;
}

/* ---- host memory-system probes for bench.py's host roofline (not a paper variant) -------------
 * STREAM-style, all OpenMP threads, each over its contiguous share: copy (read n + write n bytes,
 * non-temporal-friendly 32-B vectors) and read (sum of u64). Return bytes moved per second. */
double mt_stream_copy(const uint8_t* src, uint8_t* dst, uint64_t n, int reps) {
  double best = 0;
  for (int r = 0; r < reps; ++r) {
    const double t0 = omp_get_wtime();
#pragma omp parallel
    {
      const int T = omp_get_num_threads(), t = omp_get_thread_num();
      const uint64_t lo = n * t / T / 64 * 64, hi = (t + 1 == T) ? n : n * (t + 1) / T / 64 * 64;
      memcpy(dst + lo, src + lo, hi - lo);
    }
    const double dt = omp_get_wtime() - t0;
    if (2.0 * n / dt > best) best = 2.0 * n / dt;
  }
  return best;
}

double mt_stream_read(const uint8_t* src, uint64_t n, int reps, uint64_t* sink) {
  double best = 0;
  uint64_t acc = 0;
  for (int r = 0; r < reps; ++r) {
    const double t0 = omp_get_wtime();
#pragma omp parallel reduction(+ : acc)
    {
      const int T = omp_get_num_threads(), t = omp_get_thread_num();
      const uint64_t lo = n / 8 * t / T, hi = n / 8 * (t + 1) / T;
      const uint64_t* p = (const uint64_t*)src;
      uint64_t a0 = 0, a1 = 0, a2 = 0, a3 = 0;
      uint64_t i = lo;
      for (; i + 4 <= hi; i += 4) { a0 += p[i]; a1 += p[i + 1]; a2 += p[i + 2]; a3 += p[i + 3]; }
      for (; i < hi; ++i) a0 += p[i];
      acc += a0 + a1 + a2 + a3;
    }
    const double dt = omp_get_wtime() - t0;
    if (1.0 * n / dt > best) best = 1.0 * n / dt;
  }
  *sink = acc;
  return best;
}
