/* oracle.c — CPU ORACLE (TEST INFRASTRUCTURE ONLY; see oracle.h for who may call it).
 *
 * A plain, slow, obviously correct per-walk loop. Every function cites the passage it follows.
 * No blocking, batching, partitioning or reordering: walks are independent (PAPER.md:395,
 * "embarrassingly parallel"), so the only parallelism is an OpenMP loop over walk IDs, which
 * cannot change any walk's draws.
 */
#include "oracle.h"
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

/* ---- Philox4x32-10 (reading R3; Salmon, Moraes, Dror, Shaw, SC'11, "Parallel random numbers:
 * as easy as 1, 2, 3"; constants as published with Random123). ---- */
#define PHILOX_M0 0xD2511F53u
#define PHILOX_M1 0xCD9E8D57u
#define PHILOX_W0 0x9E3779B9u
#define PHILOX_W1 0xBB67AE85u

void oracle_philox4x32_10(const uint32_t ctr_in[4], const uint32_t key_in[2], uint32_t out[4]) {
  uint32_t c[4] = {ctr_in[0], ctr_in[1], ctr_in[2], ctr_in[3]};
  uint32_t k[2] = {key_in[0], key_in[1]};
  for (int round = 0; round < 10; ++round) {
    if (round > 0) { /* key schedule: bump by the Weyl constants between rounds */
      k[0] += PHILOX_W0;
      k[1] += PHILOX_W1;
    }
    uint64_t p0 = (uint64_t)PHILOX_M0 * (uint64_t)c[0];
    uint64_t p1 = (uint64_t)PHILOX_M1 * (uint64_t)c[2];
    uint32_t hi0 = (uint32_t)(p0 >> 32), lo0 = (uint32_t)p0;
    uint32_t hi1 = (uint32_t)(p1 >> 32), lo1 = (uint32_t)p1;
    uint32_t n0 = hi1 ^ c[1] ^ k[0];
    uint32_t n1 = lo1;
    uint32_t n2 = hi0 ^ c[3] ^ k[1];
    uint32_t n3 = lo0;
    c[0] = n0; c[1] = n1; c[2] = n2; c[3] = n3;
  }
  out[0] = c[0]; out[1] = c[1]; out[2] = c[2]; out[3] = c[3];
}

/* blk(w,t,j) = Philox(ctr = {t, j, w_lo, w_hi}, key = {seed_lo, seed_hi})  (reading R3) */
static void blk(uint64_t seed, uint64_t w, uint32_t t, uint32_t j, uint32_t out[4]) {
  uint32_t ctr[4] = {t, j, (uint32_t)w, (uint32_t)(w >> 32)};
  uint32_t key[2] = {(uint32_t)seed, (uint32_t)(seed >> 32)};
  oracle_philox4x32_10(ctr, key, out);
}

/* PPR coin threshold (reading R5): T = floor(alpha * 2^32), terminate iff x0 < T. */
uint32_t oracle_ppr_threshold(double alpha) {
  double t = alpha * 4294967296.0;
  if (!(t >= 0.0)) return 0;
  if (t >= 4294967295.0) return 0xFFFFFFFFu;
  return (uint32_t)t; /* truncation == floor for t >= 0 */
}

/* Lemire, "Fast random integer generation in an interval", TOMACS 2019 (reading R4):
 * with m = x*d (64-bit), accept iff the low word of m is >= (2^32 mod d); the index is m >> 32.
 * Accepted words map to each residue exactly floor(2^32/d) times (pin P4). */
int oracle_lemire_accept(uint32_t x, uint32_t d, uint32_t* idx) {
  uint64_t m = (uint64_t)x * (uint64_t)d;
  uint32_t low = (uint32_t)m;
  uint32_t threshold = (uint32_t)((1ULL << 32) % (uint64_t)d);
  if (low >= threshold) {
    *idx = (uint32_t)(m >> 32);
    return 1;
  }
  return 0;
}

/* Word stream of step (w,t): blk(w,t,0).x1, .x2, .x3, blk(w,t,1).x0..x3, blk(w,t,2).x0..x3, ...
 * (x0 of block 0 is the PPR coin; reading R3). */
uint32_t oracle_lemire(uint64_t seed, uint64_t w, uint32_t t, uint32_t d, uint32_t* words_used) {
  uint32_t used = 0;
  for (uint32_t j = 0;; ++j) {
    uint32_t b[4];
    blk(seed, w, t, j, b);
    for (int i = (j == 0 ? 1 : 0); i < 4; ++i) {
      uint32_t idx;
      ++used;
      if (oracle_lemire_accept(b[i], d, &idx)) {
        if (words_used) *words_used = used;
        return idx;
      }
    }
  }
}

/* One walk, SURVEY.md §8(c) "Definition" (+ PageRank, reading R23):
 *   v = start; path[0] = v; t = 0
 *   loop: DeepWalk and t == l -> stop ("walked steps reaches l"; reading R1)
 *         PPR and t == L_max -> stop, truncated (reading R6)
 *         PPR and blk(w,t,0).x0 < T -> stop (terminate with probability p before moving; R2, R5)
 *         d = deg(v); d == 0 -> stop (dead end; reading R9)
 *         v = col[row_ptr[v] + lemire(d)]  (uniform neighbour); t += 1; path[t] = v
 *   PageRank ("at each step, a walk has a probability p to restart at a random vertex,
 *   instead of uniformly selecting one of the neighbors"): stop when t == l; if blk(w,t,0).x0 < T the
 *   step goes to vertex lemire(n) (same word stream), else to a uniform neighbour as above.
 */
uint32_t oracle_walk(uint32_t n, const uint64_t* row_ptr, const uint32_t* col, uint64_t w, uint32_t start,
                     int app, uint32_t length, uint32_t T, uint32_t lmax, uint64_t seed,
                     uint32_t* path, int* truncated) {
  uint32_t v = start;
  uint32_t t = 0;
  path[0] = v;
  *truncated = 0;
  for (;;) {
    if ((app == ORACLE_DEEPWALK || app == ORACLE_PAGERANK) && t == length) break;
    if (app == ORACLE_PPR && t == lmax) { *truncated = 1; break; }
    if (app == ORACLE_PPR) {
      uint32_t b[4];
      blk(seed, w, t, 0, b);
      if (b[0] < T) break;
    }
    if (app == ORACLE_PAGERANK) {
      uint32_t b[4];
      blk(seed, w, t, 0, b);
      if (b[0] < T) {  /* restart at a uniform random vertex */
        v = oracle_lemire(seed, w, t, n, NULL);
        t += 1;
        path[t] = v;
        continue;
      }
    }
    uint64_t d = row_ptr[v + 1] - row_ptr[v];
    if (d == 0) break;
    uint32_t i = oracle_lemire(seed, w, t, (uint32_t)d, NULL);
    v = col[row_ptr[v] + i];
    t += 1;
    path[t] = v;
  }
  return t + 1;
}

uint64_t oracle_walks(uint32_t n, const uint64_t* row_ptr, const uint32_t* col, uint64_t count,
                      const uint64_t* ids, const uint32_t* starts, int app, uint32_t length,
                      uint32_t T, uint32_t lmax, uint64_t seed, uint32_t* paths, uint32_t stride,
                      uint32_t* lengths, uint64_t* truncated, int threads) {
  uint64_t steps = 0, trunc = 0;
#ifdef _OPENMP
  if (threads > 0) omp_set_num_threads(threads);
#else
  (void)threads;
#endif
#pragma omp parallel for schedule(dynamic, 4096) reduction(+ : steps, trunc)
  for (int64_t i = 0; i < (int64_t)count; ++i) {
    uint64_t w = ids ? ids[i] : (uint64_t)i;
    uint32_t* row = paths + (uint64_t)i * stride;
    for (uint32_t s = 0; s < stride; ++s) row[s] = ORACLE_EMPTY;
    int tr = 0;
    uint32_t len = oracle_walk(n, row_ptr, col, w, starts[i], app, length, T, lmax, seed, row, &tr);
    lengths[i] = len;
    steps += len - 1;
    trunc += (uint64_t)tr;
  }
  if (truncated) *truncated = trunc;
  return steps;
}

void oracle_visit_counts(uint64_t count, const uint32_t* paths, uint32_t stride, const uint32_t* lengths,
                         uint64_t* counts) {
  for (uint64_t r = 0; r < count; ++r)
    for (uint32_t t = 0; t < lengths[r]; ++t) counts[paths[r * stride + t]] += 1;
}

void oracle_lemire_exhaustive(uint32_t d, uint64_t* hist, uint64_t* rejected, int threads) {
#ifdef _OPENMP
  if (threads > 0) omp_set_num_threads(threads);
#else
  (void)threads;
#endif
  uint64_t rej = 0;
  memset(hist, 0, sizeof(uint64_t) * d);
#pragma omp parallel reduction(+ : rej)
  {
    uint64_t* local = (uint64_t*)calloc(d, sizeof(uint64_t));
#pragma omp for schedule(static)
    for (int64_t x = 0; x < (int64_t)(1ULL << 32); ++x) {
      uint32_t idx;
      if (oracle_lemire_accept((uint32_t)x, d, &idx)) local[idx]++;
      else rej++;
    }
#pragma omp critical
    for (uint32_t i = 0; i < d; ++i) hist[i] += local[i];
    free(local);
  }
  *rejected = rej;
}
