/* oracle.h — CPU oracle for the BigKernel hot path (TEST INFRASTRUCTURE ONLY).
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference leg
 * may load this library. The product path (libbk.so and its Python binding) never links,
 * imports or calls it, and shares no code with it: the only common input is gen/.
 *
 * BigKernel reorganises WHERE, WHEN and IN WHAT LAYOUT bytes move; the computation is the
 * original kernel (§III stage 4; §VI "the same kernel"). So each
 * benchmark oracle is the plain, single-threaded definition over the whole data set in
 * record order. oracle_layout pins the staged bytes (stage 2,
 * buf[counter][tid]) generalised to 16-byte words (SURVEY O-L).
 *
 * Records ("segments"): record i = bytes [off[i], off[i+1]) with off[n] := nbytes,
 * or, when off == NULL, fixed records of rec_size bytes.
 *
 * Parity status per function: see DESIGN.md §Oracle. All functions are pinned by tests in
 * tests/test_oracle_*.py (brute force, closed forms, invariants, the paper's pattern example).
 */
#ifndef BK_ORACLE_H
#define BK_ORACLE_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

/* O1 word count (§V; central table). Word = maximal run of bytes not in
 * {0x20,0x09,0x0A,0x0B,0x0C,0x0D} inside one record (A10, A19). Writes the distinct words in
 * memcmp order (shorter prefix first): offset of the first occurrence, length, count.
 * Returns V (number of distinct words) or -(V) if V > cap (nothing valid written). */
int64_t oracle_wc(const uint8_t* text, uint64_t nbytes, const uint64_t* off, uint64_t n,
                  uint64_t* word_off, uint32_t* word_len, uint64_t* word_cnt, uint64_t cap);

/* O2 grep (MCA analogue P:965-978): key = rec[16 .. 16+strnlen(rec+16,32)); match iff the
 * pattern occurs in the key as a contiguous substring (empty pattern matches all). Records
 * shorter than 48 bytes are invalid (returns -1). Writes ascending indices (+first) into idx
 * (up to cap) and returns the match count. */
int64_t oracle_grep(const uint8_t* d, uint64_t nbytes, const uint64_t* off, uint64_t n,
                    const uint8_t* pat, uint32_t plen, uint64_t first, uint64_t* idx, uint64_t cap);

/* O3 k-means assignment + partial sums (§III.A clusterKernel / findClosestCluster;
 * P:904-909). dist_k = fp32 fmaf chain over j ascending of (x_j - mu_kj)^2; cid = argmin,
 * ties to the lowest k. count[k] (u64), sum[k*16+j] = sum of (double)x_ij over cid_i = k,
 * chk = sum_i mix64(((first+i)<<8) ^ cid_i) mod 2^64. cid may be NULL. */
void oracle_kmeans(const float* x, uint64_t n, const float* mu, uint32_t K, uint64_t first,
                   uint64_t* count, double* sum, uint64_t* chk, int32_t* cid);

/* O4 hash partition (paper target class "partition"): bucket =
 * mix64(key) >> (64 - log2 B); stable counting sort. kv = n x {u64 key, u64 value}.
 * Writes boff[0..B] and out (n x 16 B). B must be a power of two <= 2^16. Returns 0/-1. */
int oracle_partition(const uint64_t* kv, uint64_t n, uint32_t B, uint64_t* boff, uint64_t* out);

/* O5 group-by sum ("aggregate"): records {u32 key, u32 qty, f64 amount} at byte
 * stride `stride`; per key < G: count, sum qty (u64), sum amount (f64, record order).
 * Returns 0, or -1 if a key >= G. */
int oracle_groupby(const uint8_t* recs, uint64_t n, uint32_t stride, uint32_t G,
                   uint64_t* count, uint64_t* qty, double* amount);

/* O6 k-mer counting (NEXT f4; DNA assembly's k-mer table, Table I): for every
 * record the sequence field rec[seq_off .. seq_off+seq_len), every window of k consecutive bases
 * in {A,C,G,T} (a base outside the set breaks windows) is the 2-bit value sum code(b_j) 4^(k-1-j),
 * A=0 C=1 G=2 T=3. Writes the distinct k-mers ascending with their counts; returns V or -V if
 * V > cap. 1 <= k <= 31. */
int64_t oracle_kmer(const uint8_t* recs, uint64_t n, uint32_t rec_size, uint32_t seq_off, uint32_t seq_len,
                    uint32_t k, uint64_t* kmer, uint64_t* count, uint64_t cap);

/* ---- O-L: staged layout (stage 1 address generation + stage 2 assembly) ----
 * Access spec: n_ext == 0 means the WHOLE record; else n_ext extents (ext_off[e], ext_len[e])
 * relative to the record start, all inside every record (the addresses the
 * compute will touch, in access order; duplicates repeat).
 * A(lo,r) = accessed bytes of records [lo, r). */

/* Greedy chunk plan ("until addrBuf is full"; whole records only, A3):
 * chunk c = [lo_c, hi_c) with hi_c the largest r <= n such that A(lo_c, r) <= budget.
 * Writes chunk starts bounds[0..C] (bounds[C] = n). Returns C, -1 if a record exceeds the
 * budget (BK_E_RANGE), -2 if cap too small. */
int64_t oracle_plan_chunks(const uint64_t* off, uint64_t n, uint64_t nbytes, uint64_t rec_size,
                           uint32_t n_ext, const uint32_t* ext_off, const uint32_t* ext_len,
                           uint64_t budget, uint64_t* bounds, uint64_t cap);

/* Lanes of chunk [lo,hi) (each thread owns a contiguous record range):
 * first(t) = min{ r in [lo,hi] : A(lo,r) >= floor(t * A(lo,hi) / L) }, first(L) = hi.
 * Layout: S_t = accessed bytes of lane t's records in record order, W_t = ceil(|S_t|/16),
 * K_w = max W_t over warp tile w (lanes 32w..32w+31), tile_base(w) = 512 * sum_{w'<w} K_w',
 * word k of lane t at tile_base(t/32) + (k*32 + t%32)*16; holes are zero.
 * Writes lane_first[L], lane_nrec[L], lane_bytes[L] and the staged bytes (if stage != NULL,
 * cap bytes). Returns the staged size (512 * sum K_w) or -1 on error. L % 32 == 0. */
int64_t oracle_layout(const uint8_t* d, const uint64_t* off, uint64_t n, uint64_t nbytes,
                      uint64_t rec_size, uint32_t n_ext, const uint32_t* ext_off, const uint32_t* ext_len,
                      uint64_t lo, uint64_t hi, uint32_t L,
                      uint64_t* lane_first, uint64_t* lane_nrec, uint64_t* lane_bytes,
                      uint8_t* stage, uint64_t cap);

/* O-P pattern recognition (§IV.A, example P:732-734): smallest period p <= pmax
 * with a[k+1]-a[k] == strides[k mod p] for all k, confirmed by at least one delta past
 * the first period (n-1 > p: 'verifies that each subsequently generated address follows'). Returns p (base = a[0]) or 0. */
int oracle_pattern(const uint64_t* a, uint32_t n, uint32_t pmax, int64_t* strides);

/* Online form of the same detector: detect on the first T addresses only ("a few
 * addresses, storing them in a private temporary address buffer"), then verify that every later
 * address follows the pattern; the first mismatch abandons it (fallback to explicit addresses).
 * Returns p or 0. */
int oracle_pattern_online(const uint64_t* a, uint64_t n, uint32_t T, uint32_t pmax, int64_t* strides);

#ifdef __cplusplus
}
#endif
#endif
