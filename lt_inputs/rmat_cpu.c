/* rmat_cpu.c — CPU (OpenMP) build of the input generator. See ltgen.h for the recipe.
 * Two passes over the counter-hashed tuples (count, then scatter) so the tuple list is never
 * stored; then per-vertex sort + dedupe, then an order-preserving compaction of zero-degree
 * vertices. */
#include "ltgen.h"
#include "ltgen_common.h"
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

void ltgen_tuple(uint32_t scale, uint64_t seed, int permute, uint64_t e, uint32_t* u, uint32_t* v) {
  ltgen_tuple_impl(scale, ltgen_key(seed), seed, permute, e, u, v);
}

static int cmp_u32(const void* a, const void* b) {
  uint32_t x = *(const uint32_t*)a, y = *(const uint32_t*)b;
  return (x > y) - (x < y);
}

static void sort_u32(uint32_t* a, uint64_t n) {
  if (n < 32) {
    for (uint64_t i = 1; i < n; ++i) {
      uint32_t x = a[i];
      uint64_t j = i;
      while (j > 0 && a[j - 1] > x) { a[j] = a[j - 1]; --j; }
      a[j] = x;
    }
  } else {
    qsort(a, (size_t)n, sizeof(uint32_t), cmp_u32);
  }
}

int ltgen_rmat_cpu(uint32_t scale, uint64_t tuples, uint64_t seed, int permute, int threads,
                   ltgen_graph* out) {
  if (!out || scale == 0 || scale > 31) return 1;
  memset(out, 0, sizeof(*out));
#ifdef _OPENMP
  if (threads > 0) omp_set_num_threads(threads);
#else
  (void)threads;
#endif
  const uint64_t N = 1ULL << scale;
  const uint64_t key = ltgen_key(seed);
  uint32_t* cnt = (uint32_t*)calloc(N, sizeof(uint32_t));
  uint64_t* off = (uint64_t*)malloc((N + 1) * sizeof(uint64_t));
  if (!cnt || !off) { free(cnt); free(off); return 2; }

  /* pass 1: degree counts of the symmetrized multigraph without self loops */
#pragma omp parallel for schedule(static)
  for (int64_t e = 0; e < (int64_t)tuples; ++e) {
    uint32_t u, v;
    ltgen_tuple_impl(scale, key, seed, permute, (uint64_t)e, &u, &v);
    if (u == v) continue;
    __atomic_fetch_add(&cnt[u], 1u, __ATOMIC_RELAXED);
    __atomic_fetch_add(&cnt[v], 1u, __ATOMIC_RELAXED);
  }
  off[0] = 0;
  for (uint64_t i = 0; i < N; ++i) off[i + 1] = off[i] + cnt[i];
  const uint64_t M0 = off[N];
  uint32_t* adj = (uint32_t*)malloc((M0 ? M0 : 1) * sizeof(uint32_t));
  uint64_t* cur = (uint64_t*)malloc(N * sizeof(uint64_t));
  if (!adj || !cur) { free(cnt); free(off); free(adj); free(cur); return 2; }
  memcpy(cur, off, N * sizeof(uint64_t));

  /* pass 2: scatter both directions (slot order is racy; the sort below fixes it) */
#pragma omp parallel for schedule(static)
  for (int64_t e = 0; e < (int64_t)tuples; ++e) {
    uint32_t u, v;
    ltgen_tuple_impl(scale, key, seed, permute, (uint64_t)e, &u, &v);
    if (u == v) continue;
    adj[__atomic_fetch_add(&cur[u], 1ULL, __ATOMIC_RELAXED)] = v;
    adj[__atomic_fetch_add(&cur[v], 1ULL, __ATOMIC_RELAXED)] = u;
  }
  free(cur);

  /* sort + dedupe each list in place; cnt[u] becomes the unique degree */
#pragma omp parallel for schedule(dynamic, 256)
  for (int64_t u = 0; u < (int64_t)N; ++u) {
    uint32_t* a = adj + off[u];
    uint64_t d = off[u + 1] - off[u];
    if (d == 0) { cnt[u] = 0; continue; }
    sort_u32(a, d);
    uint64_t k = 1;
    for (uint64_t i = 1; i < d; ++i)
      if (a[i] != a[k - 1]) a[k++] = a[i];
    cnt[u] = (uint32_t)k;
  }

  /* order-preserving relabel of non-isolated vertices */
  uint32_t* newid = (uint32_t*)malloc(N * sizeof(uint32_t));
  if (!newid) { free(cnt); free(off); free(adj); return 2; }
  uint64_t n = 0, m = 0;
  uint32_t maxd = 0, argmax = 0;
  for (uint64_t u = 0; u < N; ++u) {
    if (cnt[u]) {
      if (cnt[u] > maxd) { maxd = cnt[u]; argmax = (uint32_t)n; }
      newid[u] = (uint32_t)n++;
      m += cnt[u];
    } else {
      newid[u] = 0xFFFFFFFFu;
    }
  }
  uint64_t* row_ptr = (uint64_t*)malloc((n + 1) * sizeof(uint64_t));
  uint32_t* col = (uint32_t*)malloc((m ? m : 1) * sizeof(uint32_t));
  if (!row_ptr || !col) { free(cnt); free(off); free(adj); free(newid); free(row_ptr); free(col); return 2; }
  row_ptr[0] = 0;
  {
    uint64_t k = 0;
    for (uint64_t u = 0; u < N; ++u)
      if (cnt[u]) { row_ptr[k + 1] = row_ptr[k] + cnt[u]; ++k; }
  }
#pragma omp parallel for schedule(dynamic, 256)
  for (int64_t u = 0; u < (int64_t)N; ++u) {
    if (!cnt[u]) continue;
    const uint32_t* a = adj + off[u];
    uint32_t* dst = col + row_ptr[newid[u]];
    for (uint32_t i = 0; i < cnt[u]; ++i) dst[i] = newid[a[i]];
  }
  free(cnt); free(off); free(adj); free(newid);
  out->n = (uint32_t)n;
  out->m = m;
  out->row_ptr = row_ptr;
  out->col = col;
  out->max_deg = maxd;
  out->argmax_deg = argmax;
  return 0;
}

void ltgen_free(ltgen_graph* g) {
  if (!g) return;
  free(g->row_ptr);
  free(g->col);
  g->row_ptr = NULL;
  g->col = NULL;
}
