// lt_kernels.cu — sm_100a kernels of the partition-centric walk-update path.
//
//   k_init      a2: write path[w][0], bin each new walk into its start partition's bucket (a5)
//   k_update    a3+a4+a5: Alg. 1 re-designed for B200. A warp takes 32 records of
//               partition k's bucket (one coalesced 512-B read of 16-B records); each lane steps its
//               walk (Philox4x32-10 + Lemire; gathers of row_ptr[v], row_ptr[v+1], col[...]; path
//               store) while v stays inside [bounds[k], bounds[k+1]); terminated
//               walks record their length, walks that left are appended to the bucket of their new
//               partition with one atomic per (warp, destination) via __match_any_sync (the B200
//               version of the paper's shared-memory "local index"). The last CTA
//               to finish retires the consumed chunks (a6).
//   k_finalize  pad unused path slots with 0xFFFFFFFF (outside the timed step)
//
// Written independently of oracle/ (which is never linked or included here).
#include "lt_internal.h"

#include <algorithm>
#include <cstdio>

namespace lt {
namespace {

constexpr uint32_t kSmemBoundsCap = 8192;  // stage bounds of up to 8191 partitions (32 KB)
constexpr uint32_t kFull = 0xFFFFFFFFu;

__device__ __forceinline__ uint32_t lanemask_lt() {
  uint32_t m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

// ---- Philox4x32-10 (Salmon et al., SC'11). counter = (t, j, wid_lo, wid_hi), key = seed. -------
__device__ __forceinline__ uint4 philox10(uint4 c, uint32_t k0, uint32_t k1) {
#pragma unroll
  for (int r = 0; r < 10; ++r) {
    const uint32_t lo0 = 0xD2511F53u * c.x;
    const uint32_t hi0 = __umulhi(0xD2511F53u, c.x);
    const uint32_t lo1 = 0xCD9E8D57u * c.z;
    const uint32_t hi1 = __umulhi(0xCD9E8D57u, c.z);
    c = make_uint4(hi1 ^ c.y ^ k0, lo1, hi0 ^ c.w ^ k1, lo0);
    k0 += 0x9E3779B9u;
    k1 += 0xBB67AE85u;
  }
  return c;
}

// Lemire's nearly-divisionless rule, taken only when the fast test (low word < d) fails: accept a
// word iff its low product word >= 2^32 mod d; otherwise continue with the next word of the
// step's stream (block 0: .y .z .w; block j >= 1: .x .y .z .w).
__device__ __noinline__ uint32_t lemire_slow(uint32_t d, uint4 b0, uint32_t t, uint32_t wlo, uint32_t whi,
                                             uint32_t k0, uint32_t k1) {
  const uint32_t thr = (0u - d) % d;
  uint64_t m = (uint64_t)b0.y * d;
  if ((uint32_t)m >= thr) return (uint32_t)(m >> 32);
  m = (uint64_t)b0.z * d;
  if ((uint32_t)m >= thr) return (uint32_t)(m >> 32);
  m = (uint64_t)b0.w * d;
  if ((uint32_t)m >= thr) return (uint32_t)(m >> 32);
  for (uint32_t j = 1;; ++j) {
    const uint4 b = philox10(make_uint4(t, j, wlo, whi), k0, k1);
    m = (uint64_t)b.x * d;
    if ((uint32_t)m >= thr) return (uint32_t)(m >> 32);
    m = (uint64_t)b.y * d;
    if ((uint32_t)m >= thr) return (uint32_t)(m >> 32);
    m = (uint64_t)b.z * d;
    if ((uint32_t)m >= thr) return (uint32_t)(m >> 32);
    m = (uint64_t)b.w * d;
    if ((uint32_t)m >= thr) return (uint32_t)(m >> 32);
  }
}

// a4: upper_bound(bounds, v) - 1 over bounds[0..P]
__device__ __forceinline__ uint32_t find_partition(const uint32_t* B, uint32_t P, uint32_t v) {
  uint32_t lo = 0, hi = P;
  while (hi - lo > 1) {
    const uint32_t mid = (lo + hi) >> 1;
    if (B[mid] <= v) lo = mid; else hi = mid;
  }
  return lo;
}

// a6: chunk installation. Chunk cidx of bucket `dest` is installed exactly once, by the thread whose
// claimed position range holds the chunk's first slot (cidx * C): it pops the free stack and
// publishes the chunk in the ring slot. Every other writer into that chunk waits for the ring slot
// to be published. Installing never waits, and a waiter only waits for a chunk whose first slot lies
// at a lower position than its own claim, so the waits cannot form a cycle.
__device__ uint32_t install_chunk(const Params& p, uint32_t dest, unsigned long long cidx) {
  const Pool& pl = p.pool;
  uint32_t* slot = pl.ring + (uint64_t)dest * pl.ring_len + (cidx % pl.ring_len);
  const int idx = atomicSub(pl.free_top, 1) - 1;
  uint32_t nc = pl.num_chunks;  // trash chunk when the pool is exhausted (flagged; cannot happen when sized)
  if (idx >= 0) nc = pl.free_list[idx];
  else atomicOr(&p.ctr->err, kErrOOM);
  if (atomicExch(slot, nc) != kEmpty) atomicOr(&p.ctr->err, kErrRing);
  return nc;
}

__device__ uint32_t wait_chunk(const Params& p, uint32_t dest, unsigned long long cidx) {
  const Pool& pl = p.pool;
  const volatile uint32_t* slot = pl.ring + (uint64_t)dest * pl.ring_len + (cidx % pl.ring_len);
  uint32_t c;
  while ((c = *slot) == kEmpty) __nanosleep(32);
  return c;
}

// a5: warp-collective append of the lanes with `active` set to bucket `dest`.
__device__ __forceinline__ void insert_warp(const Params& p, bool active, uint32_t dest, uint4 rec) {
  const uint32_t act = __ballot_sync(kFull, active);
  if (act == 0 || !active) return;
  const Pool& pl = p.pool;
  const uint32_t lane = threadIdx.x & 31u;
  const unsigned long long cmask = pl.C - 1;
  if (p.insert_mode == 1) {  // "direct write" ablation: one global atomic per walk
    const unsigned long long pos = atomicAdd(pl.cursor + dest, 1ull);
    const uint32_t c = (pos & cmask) == 0 ? install_chunk(p, dest, pos >> pl.c_shift)
                                          : wait_chunk(p, dest, pos >> pl.c_shift);
    pl.slots[((uint64_t)c << pl.c_shift) | (pos & cmask)] = rec;
    return;
  }
  const uint32_t grp = __match_any_sync(act, dest);
  const uint32_t leader = __ffs(grp) - 1;
  const uint32_t rank = __popc(grp & lanemask_lt());
  unsigned long long base = 0;
  uint32_t c0 = 0, c1 = 0;
  if (lane == leader) {
    const uint32_t cnt = __popc(grp);  // cnt <= 32 <= C: the range touches at most two chunks
    base = atomicAdd(pl.cursor + dest, (unsigned long long)cnt);
    const unsigned long long ci0 = base >> pl.c_shift, ci1 = (base + cnt - 1) >> pl.c_shift;
    if (ci1 != ci0) c1 = install_chunk(p, dest, ci1);  // chunk ci1 starts inside our range
    c0 = (base & cmask) == 0 ? install_chunk(p, dest, ci0) : wait_chunk(p, dest, ci0);
    if (ci1 == ci0) c1 = c0;
  }
  base = __shfl_sync(act, base, leader);
  c0 = __shfl_sync(act, c0, leader);
  c1 = __shfl_sync(act, c1, leader);
  const unsigned long long pos = base + rank;
  const uint32_t c = ((pos >> pl.c_shift) == (base >> pl.c_shift)) ? c0 : c1;
  pl.slots[((uint64_t)c << pl.c_shift) | (pos & cmask)] = rec;
}

__device__ __forceinline__ unsigned long long warp_sum(unsigned long long x) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(kFull, x, o);
  return x;
}

// Retire after the last CTA of a launch over bucket k: free the chunks wholly below the consumed
// position `tail` (back onto the free stack, ring slots emptied) and advance head[k] (a6).
__device__ void last_cta_retire(const Params& p, int k, unsigned long long head, unsigned long long tail) {
  __shared__ bool s_last;
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    const uint32_t ticket = atomicAdd(&p.ctr->done_ctas, 1u);
    s_last = (ticket == gridDim.x - 1);
  }
  __syncthreads();
  if (!s_last) return;
  __threadfence();
  const Pool& pl = p.pool;
  if (k >= 0 && tail > head) {
    const unsigned long long cb = head >> pl.c_shift, ce = tail >> pl.c_shift;
    for (unsigned long long ci = cb + threadIdx.x; ci < ce; ci += blockDim.x) {
      uint32_t* slot = pl.ring + (uint64_t)k * pl.ring_len + (ci % pl.ring_len);
      const uint32_t c = *(volatile uint32_t*)slot;
      *(volatile uint32_t*)slot = kEmpty;
      const int idx = atomicAdd(pl.free_top, 1);
      if (idx >= 0 && c < pl.num_chunks) pl.free_list[idx] = c;
    }
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    if (k >= 0) {
      pl.head[k] = tail;
      atomicAdd(&p.ctr->visits, tail - head);
    }
    *(volatile uint32_t*)&p.ctr->done_ctas = 0;
    __threadfence();
  }
}

__device__ __forceinline__ const uint32_t* stage_bounds(const Walk& wk, uint32_t* s_bounds) {
  if (wk.P + 1 <= kSmemBoundsCap) {
    for (uint32_t i = threadIdx.x; i <= wk.P; i += blockDim.x) s_bounds[i] = wk.bounds[i];
    __syncthreads();
    return s_bounds;
  }
  return wk.bounds;
}

// ------------------------------------------------------------------------------------------ a2
__global__ void __launch_bounds__(256) k_init(Params p, const uint32_t* __restrict__ starts, uint64_t W) {
  extern __shared__ uint32_t s_bounds[];
  const Walk& wk = p.wk;
  const uint32_t* B = stage_bounds(wk, s_bounds);
  const uint32_t lane = threadIdx.x & 31u;
  const uint64_t nwarps = (uint64_t)gridDim.x * (blockDim.x >> 5);
  for (uint64_t base = ((uint64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) * 32; base < W;
       base += nwarps * 32) {
    const uint64_t i = base + lane;
    const bool have = i < W;
    uint4 rec = make_uint4(0, 0, 0, 0);
    uint32_t dest = 0;
    if (have) {
      const uint32_t v = starts[i];
      wk.paths[i * wk.stride] = v;
      rec = make_uint4((uint32_t)i, v, 0u, 0u);
      dest = find_partition(B, wk.P, v);
    }
    insert_warp(p, have, dest, rec);
  }
  last_cta_retire(p, -1, 0, 0);
}

// ------------------------------------------------------------------------------- a3 + a4 + a5
template <int APP>
__global__ void __launch_bounds__(256, 4) k_update(Params p, uint32_t k) {
  extern __shared__ uint32_t s_bounds[];
  const Walk& wk = p.wk;
  const Pool& pl = p.pool;
  const uint32_t* B = stage_bounds(wk, s_bounds);
  const unsigned long long head = pl.head[k];
  const unsigned long long tail = pl.cursor[k];  // no appends to bucket k during its own launch
  const uint32_t lo = wk.bounds[k];
  const uint32_t span = wk.bounds[k + 1] - lo;
  const uint32_t lane = threadIdx.x & 31u;
  const uint64_t nwarps = (uint64_t)gridDim.x * (blockDim.x >> 5);
  const uint32_t* ring_k = pl.ring + (uint64_t)k * pl.ring_len;
  unsigned long long my_steps = 0, my_trunc = 0;

  for (unsigned long long base = head + ((uint64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) * 32;
       base < tail; base += nwarps * 32) {
    const unsigned long long pos = base + lane;
    const bool have = pos < tail;
    uint4 rec = make_uint4(0, 0, 0, 0);
    bool left = false;
    uint32_t dest = 0;
    if (have) {
      const uint32_t c = ring_k[(pos >> pl.c_shift) % pl.ring_len];
      rec = __ldcs(pl.slots + (((uint64_t)c << pl.c_shift) | (pos & (pl.C - 1))));
      const uint32_t row = rec.x;
      uint32_t v = rec.y, t = rec.z;
      const uint64_t wid = wk.first_walk_id + row;
      const uint32_t wlo = (uint32_t)wid, whi = (uint32_t)(wid >> 32);
      uint32_t* prow = wk.paths + (uint64_t)row * wk.stride;
      bool trunc = false;
      for (;;) {
        if (APP == 0) {
          if (t == wk.length) break;
        } else {
          if (t == wk.lmax) { trunc = true; break; }
        }
        const uint4 b = philox10(make_uint4(t, 0u, wlo, whi), wk.seed_lo, wk.seed_hi);
        if (APP == 1 && b.x < wk.T) break;
        const unsigned long long off = __ldg(wk.row_ptr + v);
        const unsigned long long end = __ldg(wk.row_ptr + v + 1);
        const uint32_t d = (uint32_t)(end - off);
        if (d == 0) break;
        const uint64_t m = (uint64_t)b.y * d;
        const uint32_t idx = ((uint32_t)m < d) ? lemire_slow(d, b, t, wlo, whi, wk.seed_lo, wk.seed_hi)
                                               : (uint32_t)(m >> 32);
        v = __ldg(wk.col + off + idx);
        ++t;
        prow[t] = v;
        if (v - lo >= span) { left = true; break; }
      }
      if (left) {
        dest = find_partition(B, wk.P, v);
        rec.y = v;
        rec.z = t;
      } else {
        wk.lengths[row] = t + 1;
        my_steps += t;
        my_trunc += trunc ? 1 : 0;
      }
    }
    insert_warp(p, left, dest, rec);
  }
  my_steps = warp_sum(my_steps);
  my_trunc = warp_sum(my_trunc);
  if (lane == 0 && my_steps) atomicAdd(&p.ctr->steps, my_steps);
  if (lane == 0 && my_trunc) atomicAdd(&p.ctr->truncated, my_trunc);
  last_cta_retire(p, (int)k, head, tail);
}

// ---------------------------------------------------------------------------- output helpers
__global__ void k_finalize(Params p, uint64_t W) {
  const Walk& wk = p.wk;
  const uint32_t lane = threadIdx.x & 31u;
  const uint64_t nwarps = (uint64_t)gridDim.x * (blockDim.x >> 5);
  for (uint64_t base = ((uint64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) * 32; base < W;
       base += nwarps * 32) {
    const uint32_t L = (base + lane < W) ? wk.lengths[base + lane] : (uint32_t)wk.stride;
    uint32_t todo = __ballot_sync(kFull, L < wk.stride);
    while (todo) {
      const int j = __ffs(todo) - 1;
      todo &= todo - 1;
      const uint32_t Lj = __shfl_sync(kFull, L, j);
      uint32_t* prow = wk.paths + (base + j) * wk.stride;
      for (uint64_t t = Lj + lane; t < wk.stride; t += 32) prow[t] = kEmpty;
    }
  }
}

__global__ void k_gather_rows(Params p, const unsigned long long* rows, uint64_t count, uint32_t* out,
                              uint32_t* out_len) {
  const Walk& wk = p.wk;
  const uint64_t total = count * wk.stride;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total;
       i += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t r = i / wk.stride, t = i % wk.stride;
    out[i] = wk.paths[rows[r] * wk.stride + t];
    if (t == 0) out_len[r] = wk.lengths[rows[r]];
  }
}

__global__ void k_check_range(const uint32_t* a, uint64_t cnt, uint32_t n, uint32_t* bad) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < cnt; i += (uint64_t)gridDim.x * blockDim.x)
    if (a[i] >= n) { atomicOr(bad, 1u); return; }
}

__global__ void k_pool_reset(Params p) {
  const Pool& pl = p.pool;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  const uint64_t tid = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  for (uint64_t i = tid; i < pl.num_chunks; i += stride) pl.free_list[i] = (uint32_t)i;
  const uint64_t nring = (uint64_t)p.wk.P * pl.ring_len;
  for (uint64_t i = tid; i < nring; i += stride) pl.ring[i] = kEmpty;
  for (uint64_t i = tid; i < p.wk.P; i += stride) { pl.head[i] = 0; pl.cursor[i] = 0; }
  if (tid == 0) {
    *pl.free_top = (int)pl.num_chunks;
    p.ctr->steps = 0; p.ctr->visits = 0; p.ctr->truncated = 0; p.ctr->err = 0; p.ctr->done_ctas = 0;
  }
}

inline size_t bounds_smem(const Params& p) {
  return (p.wk.P + 1 <= kSmemBoundsCap) ? (size_t)(p.wk.P + 1) * sizeof(uint32_t) : 0;
}

int g_num_sms = 0;
int num_sms() {
  if (!g_num_sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&g_num_sms, cudaDevAttrMultiProcessorCount, dev);
    if (g_num_sms <= 0) g_num_sms = 148;
  }
  return g_num_sms;
}

}  // namespace

uint32_t update_smem_bounds_cap() { return kSmemBoundsCap - 1; }

int update_kernel_occupancy(uint32_t block) {
  int nb = 0;
  cudaFuncSetAttribute(k_update<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, kSmemBoundsCap * 4);
  cudaFuncSetAttribute(k_update<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, kSmemBoundsCap * 4);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_update<0>, (int)block, 0);
  return nb > 0 ? nb : 1;
}

cudaError_t launch_init(const Params& p, const uint32_t* starts, uint64_t W, cudaStream_t s) {
  uint64_t want = (W + 255) / 256;
  uint32_t grid = (uint32_t)std::min<uint64_t>(want ? want : 1, (uint64_t)num_sms() * 8);
  cudaFuncSetAttribute(k_init, cudaFuncAttributeMaxDynamicSharedMemorySize, kSmemBoundsCap * 4);
  k_init<<<grid, 256, bounds_smem(p), s>>>(p, starts, W);
  return cudaGetLastError();
}

cudaError_t launch_update(const Params& p, uint32_t k, uint32_t grid, uint32_t block, cudaStream_t s) {
  if (p.wk.app == 0) k_update<0><<<grid, block, bounds_smem(p), s>>>(p, k);
  else k_update<1><<<grid, block, bounds_smem(p), s>>>(p, k);
  return cudaGetLastError();
}

cudaError_t launch_finalize_paths(const Params& p, uint64_t W, cudaStream_t s) {
  uint64_t want = (W + 255) / 256;
  uint32_t grid = (uint32_t)std::min<uint64_t>(want ? want : 1, (uint64_t)num_sms() * 8);
  k_finalize<<<grid, 256, 0, s>>>(p, W);
  return cudaGetLastError();
}

cudaError_t launch_gather_rows(const Params& p, const unsigned long long* rows, uint64_t count,
                               uint32_t* out_paths, uint32_t* out_lengths, cudaStream_t s) {
  uint64_t want = (count * p.wk.stride + 255) / 256;
  uint32_t grid = (uint32_t)std::min<uint64_t>(want ? want : 1, (uint64_t)num_sms() * 8);
  k_gather_rows<<<grid, 256, 0, s>>>(p, rows, count, out_paths, out_lengths);
  return cudaGetLastError();
}

cudaError_t launch_check_col(const uint32_t* col, uint64_t m, uint32_t n, uint32_t* bad, cudaStream_t s) {
  if (!m) return cudaSuccess;
  k_check_range<<<num_sms() * 4, 256, 0, s>>>(col, m, n, bad);
  return cudaGetLastError();
}

cudaError_t launch_check_starts(const uint32_t* starts, uint64_t W, uint32_t n, uint32_t* bad, cudaStream_t s) {
  if (!W) return cudaSuccess;
  k_check_range<<<num_sms() * 4, 256, 0, s>>>(starts, W, n, bad);
  return cudaGetLastError();
}

cudaError_t launch_pool_reset(const Params& p, cudaStream_t s) {
  k_pool_reset<<<num_sms() * 4, 256, 0, s>>>(p);
  return cudaGetLastError();
}

}  // namespace lt
