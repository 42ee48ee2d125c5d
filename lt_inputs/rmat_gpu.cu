// rmat_gpu.cu — GPU build of the input generator (same recipe and bit-identical output as
// rmat_cpu.c; see ltgen.h). Used by bench.py for the scale-26 workloads, where the CPU build
// would take minutes. Input generation only: none of the random-walk method lives here.
//
//   1. each tuple e -> two 2*scale-bit keys (u<<scale|v), (v<<scale|u); self loops -> sentinel
//   2. cub radix sort of the keys (64-bit item count)
//   3. dedupe: keep key[i] != key[i-1] (sentinel dropped), count unique degrees per vertex
//   4. order-preserving relabel of non-isolated vertices (exclusive scan of nz flags)
//   5. row_ptr = exclusive scan of compacted degrees; col[i] = newid[v of i-th kept key]
#include "ltgen.h"
#include "ltgen_common.h"
#include <cub/cub.cuh>
#include <cuda_runtime.h>
#include <stdio.h>
#include <string>

static thread_local std::string g_err;

#define GCHECK(x)                                                                  \
  do {                                                                             \
    cudaError_t _e = (x);                                                          \
    if (_e != cudaSuccess) {                                                       \
      g_err = std::string(#x) + ": " + cudaGetErrorString(_e);                     \
      rc = 3;                                                                      \
      goto done;                                                                   \
    }                                                                              \
  } while (0)

__global__ void k_make_keys(uint32_t scale, uint64_t key, uint64_t seed, int permute,
                            uint64_t tuples, uint64_t sentinel, uint64_t* keys) {
  uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t e = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; e < tuples; e += stride) {
    uint32_t u, v;
    ltgen_tuple_impl(scale, key, seed, permute, e, &u, &v);
    uint64_t a = sentinel, b = sentinel;
    if (u != v) {
      a = ((uint64_t)u << scale) | v;
      b = ((uint64_t)v << scale) | u;
    }
    keys[2 * e] = a;
    keys[2 * e + 1] = b;
  }
}

__global__ void k_flags(const uint64_t* keys, uint64_t num, uint64_t sentinel, uint32_t scale,
                        uint8_t* keep, uint32_t* deg) {
  uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < num; i += stride) {
    uint64_t k = keys[i];
    bool kp = (k != sentinel) && (i == 0 || keys[i - 1] != k);
    keep[i] = kp ? 1 : 0;
    if (kp) atomicAdd(&deg[(uint32_t)(k >> scale)], 1u);
  }
}

__global__ void k_nz(const uint32_t* deg, uint64_t N, uint32_t* nz) {
  uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < N; i += stride)
    nz[i] = deg[i] ? 1u : 0u;
}

__global__ void k_compact_deg(const uint32_t* deg, const uint32_t* newid, uint64_t N,
                              uint64_t* cdeg, unsigned long long* best) {
  uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < N; i += stride) {
    uint32_t d = deg[i];
    if (d) {
      uint32_t id = newid[i];
      cdeg[id] = d;
      // max degree, ties to the smallest new id
      unsigned long long packed = ((unsigned long long)d << 32) | (0xFFFFFFFFu - id);
      atomicMax(best, packed);
    }
  }
}

__global__ void k_col(const uint64_t* ukeys, uint64_t num, uint32_t scale, const uint32_t* newid,
                      uint32_t* col) {
  uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  uint64_t mask = (1ULL << scale) - 1ULL;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < num; i += stride)
    col[i] = newid[(uint32_t)(ukeys[i] & mask)];
}

extern "C" const char* ltgen_gpu_last_error(void) { return g_err.c_str(); }
extern "C" void ltgen_gpu_free(void* p) { if (p) cudaFree(p); }
extern "C" int ltgen_gpu_memcpy(void* dst, const void* src, uint64_t bytes) {
  cudaError_t e = cudaMemcpy(dst, src, bytes, cudaMemcpyDefault);
  if (e != cudaSuccess) { g_err = cudaGetErrorString(e); return 3; }
  return 0;
}

extern "C" int ltgen_rmat_gpu(uint32_t scale, uint64_t tuples, uint64_t seed, int permute,
                              uint32_t* n_out, uint64_t* m_out, uint64_t** d_row_ptr,
                              uint32_t** d_col, uint32_t* max_deg, uint32_t* argmax_deg) {
  int rc = 0;
  if (scale == 0 || scale > 31) { g_err = "bad scale"; return 1; }
  const uint64_t N = 1ULL << scale;
  const uint64_t K = 2 * tuples;
  const uint64_t sentinel = (1ULL << (2 * scale)) - 1ULL;  // (N-1,N-1): a self loop, never an edge
  const int end_bit = (int)(2 * scale);
  uint64_t *k0 = nullptr, *k1 = nullptr, *cdeg = nullptr, *row_ptr = nullptr;
  uint8_t* keep = nullptr;
  uint32_t *deg = nullptr, *nz = nullptr, *newid = nullptr, *col = nullptr;
  int64_t* nsel = nullptr;
  unsigned long long* best = nullptr;
  void* tmp = nullptr;
  size_t tmp_bytes = 0, need = 0;
  uint32_t n = 0;
  int64_t m = 0;
  unsigned long long hbest = 0;
  const int TB = 256, GB = 148 * 16;
  *d_row_ptr = nullptr;
  *d_col = nullptr;

  GCHECK(cudaMalloc(&k0, K * sizeof(uint64_t)));
  GCHECK(cudaMalloc(&k1, K * sizeof(uint64_t)));
  k_make_keys<<<GB, TB>>>(scale, ltgen_key(seed), seed, permute, tuples, sentinel, k0);
  GCHECK(cudaGetLastError());
  {
    cub::DoubleBuffer<uint64_t> db(k0, k1);
    GCHECK(cub::DeviceRadixSort::SortKeys(nullptr, need, db, (int64_t)K, 0, end_bit));
    GCHECK(cudaMalloc(&tmp, need));
    tmp_bytes = need;
    GCHECK(cub::DeviceRadixSort::SortKeys(tmp, tmp_bytes, db, (int64_t)K, 0, end_bit));
    if (db.Current() != k0) std::swap(k0, k1);  // k0 = sorted keys
  }
  GCHECK(cudaFree(tmp)); tmp = nullptr;
  GCHECK(cudaMalloc(&keep, K));
  GCHECK(cudaMalloc(&deg, N * sizeof(uint32_t)));
  GCHECK(cudaMemset(deg, 0, N * sizeof(uint32_t)));
  k_flags<<<GB, TB>>>(k0, K, sentinel, scale, keep, deg);
  GCHECK(cudaGetLastError());
  GCHECK(cudaMalloc(&nsel, sizeof(int64_t)));
  need = 0;
  GCHECK(cub::DeviceSelect::Flagged(nullptr, need, k0, keep, k1, nsel, (int64_t)K));
  GCHECK(cudaMalloc(&tmp, need));
  tmp_bytes = need;
  GCHECK(cub::DeviceSelect::Flagged(tmp, tmp_bytes, k0, keep, k1, nsel, (int64_t)K));
  GCHECK(cudaFree(tmp)); tmp = nullptr;
  GCHECK(cudaMemcpy(&m, nsel, sizeof(int64_t), cudaMemcpyDeviceToHost));
  GCHECK(cudaFree(k0)); k0 = nullptr;
  GCHECK(cudaFree(keep)); keep = nullptr;

  GCHECK(cudaMalloc(&nz, N * sizeof(uint32_t)));
  GCHECK(cudaMalloc(&newid, N * sizeof(uint32_t)));
  k_nz<<<GB, TB>>>(deg, N, nz);
  GCHECK(cudaGetLastError());
  need = 0;
  GCHECK(cub::DeviceScan::ExclusiveSum(nullptr, need, nz, newid, (int64_t)N));
  GCHECK(cudaMalloc(&tmp, need));
  tmp_bytes = need;
  GCHECK(cub::DeviceScan::ExclusiveSum(tmp, tmp_bytes, nz, newid, (int64_t)N));
  GCHECK(cudaFree(tmp)); tmp = nullptr;
  {
    uint32_t last_id = 0, last_nz = 0;
    GCHECK(cudaMemcpy(&last_id, newid + N - 1, 4, cudaMemcpyDeviceToHost));
    GCHECK(cudaMemcpy(&last_nz, nz + N - 1, 4, cudaMemcpyDeviceToHost));
    n = last_id + last_nz;
  }
  GCHECK(cudaMalloc(&cdeg, ((uint64_t)n + 1) * sizeof(uint64_t)));
  GCHECK(cudaMemset(cdeg, 0, ((uint64_t)n + 1) * sizeof(uint64_t)));
  GCHECK(cudaMalloc(&best, sizeof(unsigned long long)));
  GCHECK(cudaMemset(best, 0, sizeof(unsigned long long)));
  k_compact_deg<<<GB, TB>>>(deg, newid, N, cdeg, best);
  GCHECK(cudaGetLastError());
  GCHECK(cudaMalloc(&row_ptr, ((uint64_t)n + 1) * sizeof(uint64_t)));
  need = 0;
  GCHECK(cub::DeviceScan::ExclusiveSum(nullptr, need, cdeg, row_ptr, (int64_t)n + 1));
  GCHECK(cudaMalloc(&tmp, need));
  tmp_bytes = need;
  GCHECK(cub::DeviceScan::ExclusiveSum(tmp, tmp_bytes, cdeg, row_ptr, (int64_t)n + 1));
  GCHECK(cudaFree(tmp)); tmp = nullptr;
  GCHECK(cudaMalloc(&col, (m ? m : 1) * sizeof(uint32_t)));
  k_col<<<GB, TB>>>(k1, (uint64_t)m, scale, newid, col);
  GCHECK(cudaGetLastError());
  GCHECK(cudaMemcpy(&hbest, best, sizeof(hbest), cudaMemcpyDeviceToHost));
  GCHECK(cudaDeviceSynchronize());
  *n_out = n;
  *m_out = (uint64_t)m;
  *max_deg = (uint32_t)(hbest >> 32);
  *argmax_deg = 0xFFFFFFFFu - (uint32_t)(hbest & 0xFFFFFFFFu);
  *d_row_ptr = row_ptr; row_ptr = nullptr;
  *d_col = col; col = nullptr;
done:
  if (k0) cudaFree(k0);
  if (k1) cudaFree(k1);
  if (keep) cudaFree(keep);
  if (deg) cudaFree(deg);
  if (nz) cudaFree(nz);
  if (newid) cudaFree(newid);
  if (cdeg) cudaFree(cdeg);
  if (nsel) cudaFree(nsel);
  if (best) cudaFree(best);
  if (tmp) cudaFree(tmp);
  if (row_ptr) cudaFree(row_ptr);
  if (col) cudaFree(col);
  return rc;
}
