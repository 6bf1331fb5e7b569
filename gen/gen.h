/* gen.h — seeded synthetic input generators (SURVEY §8(c) "Generators", §8(d) input recipes).
 *
 * This module holds ONLY input generation: random bytes/records with the shapes of the
 * paper's workloads (Table I) and BASELINE.json's configs. It contains
 * none of the method's arithmetic (no tokenising, matching, distances, hashing of keys
 * into buckets, aggregation). Both the CUDA path's tests/bench and the oracle consume its
 * output; neither side shares any other code.
 *
 * Counter-based RNG: R(seed, stream, i) = mix64(mix64(seed ^ stream*C1) + i*C2), so any
 * record range (a shard) regenerates independently and identically.
 */
#ifndef BK_GEN_H
#define BK_GEN_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

uint64_t gen_R(uint64_t seed, uint64_t stream, uint64_t i);

/* C1 — word-count text: lines of Zipf(1.0) words from a 65,536-word vocabulary,
 * 0..16 words per line separated by single spaces, every line ends in '\n'.
 * Writes whole lines while total <= cap_bytes and lines <= cap_recs.
 * Outputs byte count and line count; off[i] = start of line i. Returns 0 on success. */
int gen_text(uint64_t seed, uint64_t cap_bytes, uint8_t* buf, uint64_t* off, uint64_t cap_recs,
             uint64_t* out_nbytes, uint64_t* out_nrec);

/* C2 — grep records (A16): [u32 len][u32 flags][u64 id][char key[32] NUL-padded][payload len-48].
 * len = 48 + 8*(R%53) in [48,464] (mean 256, 8-byte aligned); key length 8..32 lowercase;
 * "bigk" planted with p = 1/100. Records [first, first+n) of the global sequence.
 * Pass 1: gen_grep_sizes fills off[0..n) (relative to the shard start) and returns total bytes.
 * Pass 2: gen_grep_fill writes the bytes (threads: OpenMP). */
uint64_t gen_grep_sizes(uint64_t seed, uint64_t first, uint64_t n, uint64_t* off);
uint64_t gen_grep_count_for_bytes(uint64_t seed, uint64_t first, uint64_t max_bytes);
void gen_grep_fill(uint64_t seed, uint64_t first, uint64_t n, const uint64_t* off, uint8_t* buf, int threads);

/* C3 — k-means points: n x 16 fp32, 64 Gaussian-like blobs (Irwin-Hall, sigma 4) with
 * centres U[20,80)^16, so every coordinate is >= 6.1 (A13). Points [first, first+n). */
void gen_points(uint64_t seed, uint64_t first, uint64_t n, float* x, int threads);

/* C4 — key/value records {u64 key = R(seed,1,i), u64 value = i}. */
void gen_kv(uint64_t seed, uint64_t first, uint64_t n, uint64_t* kv, int threads);

/* C5 — group-by records {u32 key < G, u32 qty in [1,100], f64 amount = cents/100,
 * cents in [0,1e5)} at record stride `stride` (16 = dense; 64 = sparse, 48 B filler).
 * zipf != 0 draws keys from Zipf(1.0) over G instead of uniform. */
void gen_groupby(uint64_t seed, uint64_t first, uint64_t n, uint32_t G, uint32_t stride, int zipf,
                 uint8_t* buf, int threads);

/* f4 — DNA reads: 256-B records, 96-base sequence at +16 (ACGT, 'N' calls), sampled from a seeded
 * genome of genome_len bases with err_pm / n_pm per-mille substitution / N rates. */
void gen_dna(uint64_t seed, uint64_t first, uint64_t n, uint64_t genome_len, uint32_t err_pm, uint32_t n_pm,
             uint8_t* buf, int threads);

/* 2 MiB-aligned anonymous mapping for large data sets; huge != 0 asks for transparent huge pages
 * (madvise). Free with gen_free(base, len). */
void* gen_alloc(uint64_t bytes, int huge, void** base_out, uint64_t* len_out);
void gen_free(void* base, uint64_t len);

#ifdef __cplusplus
}
#endif
#endif
