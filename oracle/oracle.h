/* oracle.h — CPU ORACLE for the LightTraffic walk-update path. TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may
 * load this library. The product path (paper_conf_icde_xing0wxl23_b200/) never does; it shares no
 * code, header, table or constant generator with this file.
 *
 * What it computes:
 *   A walk w starts at starts[w] and moves to a uniformly chosen neighbour in each step
 *   (§II-A). DeepWalk / uniform sampling stops when walked_steps reaches l
 *   (§IV-A). PPR terminates with probability p in each step,
 *   checked BEFORE each move (reading R2), capped at L_max steps (reading R6).
 *   The RNG (reading R3) is Philox4x32-10 (Salmon et al. SC'11) keyed by the seed, with counter
 *   (t, j, w_lo, w_hi); the uniform neighbour index is Lemire's unbiased multiply-shift with
 *   rejection (reading R4) over the word stream blk(w,t,0).x1..x3, blk(w,t,1).x0..x3, ...
 *   The PPR coin is x0 < T with T = floor(alpha * 2^32) (reading R5).
 *   PageRank (reading R23): fixed length l; at each step the same coin x0 < T (T from
 *   the restart probability p) sends the walk to a uniform vertex, Lemire over n on the same word
 *   stream, instead of to a uniform neighbour.
 * Pins: tests/test_oracle_pins.py (Philox KATs, Lemire exhaustive counts, closed-form Markov and
 * PPR distributions, chi-square uniformity, geometric length, edge validity, brute force).
 */
#ifndef LT_ORACLE_H
#define LT_ORACLE_H
#include <stdint.h>

#define ORACLE_DEEPWALK 0
#define ORACLE_PPR 1
#define ORACLE_PAGERANK 2 /* random walk with restart; reading R23 */
#define ORACLE_EMPTY 0xFFFFFFFFu

void oracle_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]);
uint32_t oracle_ppr_threshold(double alpha);
/* Uniform index in [0, d) for step (w, t), d >= 1. *words_used (optional) = words consumed. */
uint32_t oracle_lemire(uint64_t seed, uint64_t w, uint32_t t, uint32_t d, uint32_t* words_used);
/* Lemire's accept rule applied to ONE word x; returns 1 and *idx on accept, 0 on reject. */
int oracle_lemire_accept(uint32_t x, uint32_t d, uint32_t* idx);

/* One walk. path has room for stride entries; returns the number of path vertices.
 * *truncated set to 1 if a PPR walk hit L_max. Unused path slots are left untouched. */
uint32_t oracle_walk(uint32_t n, const uint64_t* row_ptr, const uint32_t* col, uint64_t w, uint32_t start,
                     int app, uint32_t length, uint32_t T, uint32_t lmax, uint64_t seed,
                     uint32_t* path, int* truncated);

/* The walks with IDs ids[i] (or 0..count-1 when ids == NULL) starting at starts[i]; rows of
 * `stride` u32 in paths (unused slots = 0xFFFFFFFF); lengths[i] = path vertices. OpenMP over
 * walks with `threads` threads (0 = default). Returns total steps = sum(lengths - 1). */
uint64_t oracle_walks(uint32_t n, const uint64_t* row_ptr, const uint32_t* col, uint64_t count,
                      const uint64_t* ids, const uint32_t* starts, int app, uint32_t length,
                      uint32_t T, uint32_t lmax, uint64_t seed, uint32_t* paths, uint32_t stride,
                      uint32_t* lengths, uint64_t* truncated, int threads);

/* Visit frequency: counts[v] += number of path entries equal to v, over the
 * `count` rows of paths (row r has lengths[r] entries). */
void oracle_visit_counts(uint64_t count, const uint32_t* paths, uint32_t stride, const uint32_t* lengths,
                         uint64_t* counts);

/* Lemire exhaustive check (pin P4): over all 2^32 words x, histogram of accepted residues. */
void oracle_lemire_exhaustive(uint32_t d, uint64_t* hist, uint64_t* rejected, int threads);

#endif
