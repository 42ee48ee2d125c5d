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
#include <vector>

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

// ---------------------------------------------------------------------------------------------
// Ranged build for graphs whose key arrays do not fit in device memory at once (BASELINE configs[4],
// Kronecker scale 28, 5.5B tuples -> 11B keys): the same recipe and the same output, computed one
// source-vertex range at a time. A histogram pass counts the keys per 2^hb source-prefix bin; bins
// are grouped into ranges of at most `max_pass_keys` keys; for each range every tuple is regenerated
// and only the keys whose source lies in the range are appended, sorted and deduplicated; the
// ranges' neighbour lists concatenate in global (u, v) order. Compaction / relabel runs at the end.
static constexpr uint32_t kHistBits = 12;

__global__ void k_hist(uint32_t scale, uint64_t key, uint64_t seed, int permute, uint64_t tuples, uint32_t hb,
                       unsigned long long* hist) {
  __shared__ unsigned int sh[1u << kHistBits];
  for (uint32_t i = threadIdx.x; i < (1u << hb); i += blockDim.x) sh[i] = 0;
  __syncthreads();
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t e = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; e < tuples; e += stride) {
    uint32_t u, v;
    ltgen_tuple_impl(scale, key, seed, permute, e, &u, &v);
    if (u == v) continue;
    atomicAdd(&sh[u >> (scale - hb)], 1u);
    atomicAdd(&sh[v >> (scale - hb)], 1u);
  }
  __syncthreads();
  for (uint32_t i = threadIdx.x; i < (1u << hb); i += blockDim.x)
    if (sh[i]) atomicAdd(&hist[i], (unsigned long long)sh[i]);
}

__global__ void k_range_keys(uint32_t scale, uint64_t key, uint64_t seed, int permute, uint64_t tuples,
                             uint32_t lo, uint64_t hi, uint64_t* keys, unsigned long long* count, uint64_t cap) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  const uint64_t nt = (tuples + stride - 1) / stride * stride;  // every lane runs the same trip count
  for (uint64_t e = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; e < nt; e += stride) {
    uint32_t u = 0, v = 0;
    if (e < tuples) ltgen_tuple_impl(scale, key, seed, permute, e, &u, &v);
    const bool a = e < tuples && u != v && u >= lo && (uint64_t)u < hi;
    const bool b = e < tuples && u != v && v >= lo && (uint64_t)v < hi;
    const uint32_t na = __popc(__ballot_sync(0xFFFFFFFFu, a)), nb = __popc(__ballot_sync(0xFFFFFFFFu, b));
    const uint32_t lane = threadIdx.x & 31u;
    unsigned long long base = 0;
    if (lane == 0 && na + nb) base = atomicAdd(count, (unsigned long long)(na + nb));
    base = __shfl_sync(0xFFFFFFFFu, base, 0);
    const uint32_t lt = (1u << lane) - 1u;
    const uint32_t ra = __popc(__ballot_sync(0xFFFFFFFFu, a) & lt);
    const uint32_t rb = na + __popc(__ballot_sync(0xFFFFFFFFu, b) & lt);
    if (a && base + ra < cap) keys[base + ra] = ((uint64_t)u << scale) | v;
    if (b && base + rb < cap) keys[base + rb] = ((uint64_t)v << scale) | u;
  }
}

__global__ void k_range_flags(const uint64_t* keys, uint64_t num, uint32_t scale, uint8_t* keep, uint32_t* deg) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < num; i += stride) {
    const uint64_t k = keys[i];
    const bool kp = (i == 0 || keys[i - 1] != k);
    keep[i] = kp ? 1 : 0;
    if (kp) atomicAdd(&deg[(uint32_t)(k >> scale)], 1u);
  }
}

__global__ void k_low_bits(const uint64_t* ukeys, uint64_t num, uint32_t scale, uint32_t* col) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  const uint64_t mask = (1ULL << scale) - 1ULL;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < num; i += stride)
    col[i] = (uint32_t)(ukeys[i] & mask);
}

__global__ void k_relabel(uint32_t* col, uint64_t m, const uint32_t* newid) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < m; i += stride) col[i] = newid[col[i]];
}

extern "C" int ltgen_rmat_gpu_count(uint32_t scale, uint64_t tuples, uint64_t seed, int permute,
                                    uint64_t* keys_total, uint64_t* max_bin_keys) {
  int rc = 0;
  if (scale == 0 || scale > 31) { g_err = "bad scale"; return 1; }
  const uint32_t hb = scale < kHistBits ? scale : kHistBits;
  unsigned long long* hist = nullptr;
  std::vector<unsigned long long> h(1u << hb);
  GCHECK(cudaMalloc(&hist, sizeof(unsigned long long) << hb));
  GCHECK(cudaMemset(hist, 0, sizeof(unsigned long long) << hb));
  k_hist<<<148 * 8, 256>>>(scale, ltgen_key(seed), seed, permute, tuples, hb, hist);
  GCHECK(cudaGetLastError());
  GCHECK(cudaMemcpy(h.data(), hist, sizeof(unsigned long long) << hb, cudaMemcpyDeviceToHost));
  {
    uint64_t t = 0, mx = 0;
    for (auto x : h) { t += x; mx = x > mx ? x : mx; }
    *keys_total = t;
    if (max_bin_keys) *max_bin_keys = mx;
  }
done:
  if (hist) cudaFree(hist);
  return rc;
}

// Caller-allocated outputs: d_row_ptr holds 2^scale + 1 u64, d_col holds keys_total u32 (from
// ltgen_rmat_gpu_count). *passes receives the number of source ranges used.
extern "C" int ltgen_rmat_gpu_into(uint32_t scale, uint64_t tuples, uint64_t seed, int permute,
                                   uint64_t max_pass_keys, uint64_t* d_row_ptr, uint32_t* d_col,
                                   uint64_t col_capacity, uint32_t* n_out, uint64_t* m_out, uint32_t* max_deg,
                                   uint32_t* argmax_deg, uint32_t* passes) {
  int rc = 0;
  if (scale == 0 || scale > 31) { g_err = "bad scale"; return 1; }
  const uint64_t N = 1ULL << scale;
  const uint32_t hb = scale < kHistBits ? scale : kHistBits;
  const uint64_t key = ltgen_key(seed);
  const int TB = 256, GB = 148 * 16;
  unsigned long long *hist = nullptr, *cnt = nullptr, *best = nullptr;
  uint64_t *k0 = nullptr, *k1 = nullptr, *cdeg = nullptr;
  uint8_t* keep = nullptr;
  uint32_t *deg = nullptr, *nz = nullptr, *newid = nullptr;
  int64_t* nsel = nullptr;
  void* tmp = nullptr;
  size_t tmp_bytes = 0, need = 0;
  std::vector<unsigned long long> h(1u << hb);
  uint64_t m = 0;
  uint32_t n = 0, npass = 0;
  unsigned long long hbest = 0;
  GCHECK(cudaMalloc(&hist, sizeof(unsigned long long) << hb));
  GCHECK(cudaMemset(hist, 0, sizeof(unsigned long long) << hb));
  k_hist<<<148 * 8, 256>>>(scale, key, seed, permute, tuples, hb, hist);
  GCHECK(cudaGetLastError());
  GCHECK(cudaMemcpy(h.data(), hist, sizeof(unsigned long long) << hb, cudaMemcpyDeviceToHost));
  {
    uint64_t cap = 0;
    for (auto x : h) {
      if (x > max_pass_keys) { g_err = "a source bin exceeds max_pass_keys"; rc = 2; goto done; }
    }
    // pass buffers sized for the largest group of consecutive bins
    uint64_t acc = 0;
    for (auto x : h) {
      if (acc + x > max_pass_keys) { cap = acc > cap ? acc : cap; acc = 0; }
      acc += x;
    }
    cap = acc > cap ? acc : cap;
    if (cap == 0) cap = 1;
    GCHECK(cudaMalloc(&k0, cap * sizeof(uint64_t)));
    GCHECK(cudaMalloc(&k1, cap * sizeof(uint64_t)));
    GCHECK(cudaMalloc(&keep, cap));
    GCHECK(cudaMalloc(&cnt, sizeof(unsigned long long)));
    GCHECK(cudaMalloc(&nsel, sizeof(int64_t)));
    GCHECK(cudaMalloc(&deg, N * sizeof(uint32_t)));
    GCHECK(cudaMemset(deg, 0, N * sizeof(uint32_t)));
    need = 0;
    {
      cub::DoubleBuffer<uint64_t> db(k0, k1);
      GCHECK(cub::DeviceRadixSort::SortKeys(nullptr, need, db, (int64_t)cap, 0, (int)(2 * scale)));
    }
    {
      size_t n2 = 0;
      GCHECK(cub::DeviceSelect::Flagged(nullptr, n2, k0, keep, k1, nsel, (int64_t)cap));
      need = need > n2 ? need : n2;
    }
    GCHECK(cudaMalloc(&tmp, need));
    tmp_bytes = need;
    // walk the bins, one source range per pass
    uint32_t b0 = 0;
    const uint32_t nbins = 1u << hb;
    while (b0 < nbins) {
      uint32_t b1 = b0;
      uint64_t keys = 0;
      while (b1 < nbins && keys + h[b1] <= max_pass_keys) keys += h[b1++];
      const uint32_t lo = (uint32_t)((uint64_t)b0 << (scale - hb));
      const uint64_t hi = (uint64_t)b1 << (scale - hb);
      b0 = b1;
      if (keys == 0) continue;
      ++npass;
      GCHECK(cudaMemset(cnt, 0, sizeof(unsigned long long)));
      k_range_keys<<<GB, TB>>>(scale, key, seed, permute, tuples, lo, hi, k0, cnt, cap);
      GCHECK(cudaGetLastError());
      cub::DoubleBuffer<uint64_t> db(k0, k1);
      size_t tb = tmp_bytes;
      GCHECK(cub::DeviceRadixSort::SortKeys(tmp, tb, db, (int64_t)keys, 0, (int)(2 * scale)));
      uint64_t* sorted = db.Current();
      uint64_t* other = (sorted == k0) ? k1 : k0;
      k_range_flags<<<GB, TB>>>(sorted, keys, scale, keep, deg);
      GCHECK(cudaGetLastError());
      tb = tmp_bytes;
      GCHECK(cub::DeviceSelect::Flagged(tmp, tb, sorted, keep, other, nsel, (int64_t)keys));
      int64_t mr = 0;
      GCHECK(cudaMemcpy(&mr, nsel, sizeof(int64_t), cudaMemcpyDeviceToHost));
      if (m + (uint64_t)mr > col_capacity) { g_err = "col capacity exceeded"; rc = 2; goto done; }
      k_low_bits<<<GB, TB>>>(other, (uint64_t)mr, scale, d_col + m);
      GCHECK(cudaGetLastError());
      m += (uint64_t)mr;
    }
  }
  GCHECK(cudaFree(k0)); k0 = nullptr;
  GCHECK(cudaFree(k1)); k1 = nullptr;
  GCHECK(cudaFree(keep)); keep = nullptr;
  GCHECK(cudaFree(tmp)); tmp = nullptr;
  // compaction and relabel, as in ltgen_rmat_gpu
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
  need = 0;
  GCHECK(cub::DeviceScan::ExclusiveSum(nullptr, need, cdeg, d_row_ptr, (int64_t)n + 1));
  GCHECK(cudaMalloc(&tmp, need));
  tmp_bytes = need;
  GCHECK(cub::DeviceScan::ExclusiveSum(tmp, tmp_bytes, cdeg, d_row_ptr, (int64_t)n + 1));
  GCHECK(cudaFree(tmp)); tmp = nullptr;
  k_relabel<<<GB, TB>>>(d_col, m, newid);
  GCHECK(cudaGetLastError());
  GCHECK(cudaMemcpy(&hbest, best, sizeof(hbest), cudaMemcpyDeviceToHost));
  GCHECK(cudaDeviceSynchronize());
  *n_out = n;
  *m_out = m;
  *max_deg = (uint32_t)(hbest >> 32);
  *argmax_deg = 0xFFFFFFFFu - (uint32_t)(hbest & 0xFFFFFFFFu);
  if (passes) *passes = npass;
done:
  if (hist) cudaFree(hist);
  if (cnt) cudaFree(cnt);
  if (best) cudaFree(best);
  if (k0) cudaFree(k0);
  if (k1) cudaFree(k1);
  if (cdeg) cudaFree(cdeg);
  if (keep) cudaFree(keep);
  if (deg) cudaFree(deg);
  if (nz) cudaFree(nz);
  if (newid) cudaFree(newid);
  if (nsel) cudaFree(nsel);
  if (tmp) cudaFree(tmp);
  return rc;
}
