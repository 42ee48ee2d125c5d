/* ltgen.h — seeded synthetic graph generator (INPUT GENERATOR, not the method).
 *
 * This module produces the graphs both the CUDA path and the CPU oracle consume. It holds none
 * of the random-walk arithmetic (no Philox, no Lemire, no walk loop); its own randomness is a
 * splitmix64 counter hash, deliberately different from the walk RNG.
 *
 * Recipe (SURVEY.md §8(d) "Inputs"):
 *   - R-MAT with the Graph500 initiator (a,b,c,d) = (0.57,0.19,0.19,0.05), no noise. Tuple e draws
 *     one 32-bit word per level from splitmix64(key + 32*e + level/2) (hi word: even level,
 *     lo word: odd level); level 0 picks the most significant bit of (u,v).
 *   - "Kronecker" (permute=1): the same tuples pushed through a seeded Feistel bijection on
 *     [0, 2^scale) (cycle-walking for odd scale), Graph500-style.
 *   - Preprocessing as PAPER.md:273 (§IV-A Workload): make undirected (symmetrize), drop self
 *     loops and duplicate edges, drop zero-degree vertices with an order-preserving relabel,
 *     sort each adjacency list ascending.
 *   - Output CSR with u64 offsets and u32 neighbour IDs (the layout Table II's sizes imply,
 *     PAPER.md:277-285).
 * The output is a pure function of (scale, tuples, seed, permute): the edge SET is fixed by the
 * counter hash, and sorting fixes the order. CPU and GPU builds must therefore agree bit-exactly.
 */
#ifndef LTGEN_H
#define LTGEN_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

typedef struct ltgen_graph {
  uint32_t n;          /* vertices after compaction */
  uint64_t m;          /* directed CSR entries (= 2 x undirected edges) */
  uint64_t* row_ptr;   /* n+1, malloc'ed by the generator (CPU build) */
  uint32_t* col;       /* m */
  uint32_t max_deg;
  uint32_t argmax_deg; /* smallest ID among the max-degree vertices (PPR source) */
} ltgen_graph;

/* CPU build (OpenMP). Returns 0 on success, nonzero on bad args / OOM. Free with ltgen_free. */
int ltgen_rmat_cpu(uint32_t scale, uint64_t tuples, uint64_t seed, int permute, int threads,
                   ltgen_graph* out);
void ltgen_free(ltgen_graph* g);

/* The raw R-MAT tuple e (before any preprocessing); exposed for tests. */
void ltgen_tuple(uint32_t scale, uint64_t seed, int permute, uint64_t e, uint32_t* u, uint32_t* v);

/* GPU build (ltgen_gpu.cu): writes the same CSR into DEVICE memory it allocates with
 * cudaMalloc (caller frees with ltgen_gpu_free). Returns 0 on success. */
int ltgen_rmat_gpu(uint32_t scale, uint64_t tuples, uint64_t seed, int permute,
                   uint32_t* n, uint64_t* m, uint64_t** d_row_ptr, uint32_t** d_col,
                   uint32_t* max_deg, uint32_t* argmax_deg);
void ltgen_gpu_free(void* d_ptr);
int ltgen_gpu_memcpy(void* dst, const void* src, uint64_t bytes); /* cudaMemcpyDefault */
const char* ltgen_gpu_last_error(void);

#ifdef __cplusplus
}
#endif
#endif
