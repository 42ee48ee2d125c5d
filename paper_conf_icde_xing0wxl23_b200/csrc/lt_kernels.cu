// lt_kernels.cu — sm_100a kernels of the partition-centric walk-update path.
//
//   k_init      a2: bin each new walk into its start partition's bucket (a5); path[w][0] is written by the
//               update kernel's first sector store (or here, in the per-step path mode)
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

#include <cub/block/block_reduce.cuh>
#include <cub/block/block_scan.cuh>

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
// Records for another rank are counted into *sent_acc (a shared-memory counter of the CTA that the update
// kernels add to ctr->sent once at their end: one global atomic per group on one counter would serialise
// the peer path the way one shared cursor line did); without it straight into ctr->sent.
__device__ __forceinline__ void insert_warp(const Params& p, bool active, uint32_t dest, uint4 rec,
                                            unsigned long long* sent_acc = nullptr) {
  const uint32_t act = __ballot_sync(kFull, active);
  if (act == 0 || !active) return;
  const Pool& pl = p.pool;
  const uint32_t lane = threadIdx.x & 31u;
  const unsigned long long cmask = pl.C - 1;
  if (p.insert_mode == 1) {  // "direct write" ablation: one global atomic per walk
    const unsigned long long pos = atomicAdd(pl.cursor + (uint64_t)dest * pl.hs, 1ull);
    const uint32_t c = (pos & cmask) == 0 ? install_chunk(p, dest, pos >> pl.c_shift)
                                          : wait_chunk(p, dest, pos >> pl.c_shift);
    pl.slots[((uint64_t)c << pl.c_shift) | (pos & cmask)] = rec;
    return;
  }
  const uint32_t grp = __match_any_sync(act, dest);
  const uint32_t leader = __ffs(grp) - 1;
  const uint32_t rank = __popc(grp & lanemask_lt());
  if (p.peer.recv && dest >= p.wk.P) {  // a walk for rank q: straight into q's receive buffer (peer memory)
    const uint32_t slot = p.peer.epoch * (pl.nbuckets - p.wk.P) + (dest - p.wk.P);
    unsigned long long base = 0;
    if (lane == leader) {
      const uint32_t cnt = __popc(grp);
      base = atomicAdd(p.peer.cursor[slot], (unsigned long long)cnt);
      if (base + cnt > p.peer.cap) atomicOr(&p.ctr->err, kErrPeer);
      if (sent_acc) atomicAdd(sent_acc, (unsigned long long)cnt);
      else atomicAdd(&p.ctr->sent, (unsigned long long)cnt);
    }
    base = __shfl_sync(grp, base, leader);
    if (base + rank < p.peer.cap) p.peer.recv[slot][base + rank] = rec;
    return;
  }
  unsigned long long base = 0;
  uint32_t c0 = 0, c1 = 0;
  if (lane == leader) {
    const uint32_t cnt = __popc(grp);  // cnt <= 32 <= C: the range touches at most two chunks
    base = atomicAdd(pl.cursor + (uint64_t)dest * pl.hs, (unsigned long long)cnt);
    const unsigned long long ci0 = base >> pl.c_shift, ci1 = (base + cnt - 1) >> pl.c_shift;
    if (ci1 != ci0) c1 = install_chunk(p, dest, ci1);  // chunk ci1 starts inside our range
    c0 = (base & cmask) == 0 ? install_chunk(p, dest, ci0) : wait_chunk(p, dest, ci0);
    if (ci1 == ci0) c1 = c0;
  }
  // each lane needs only its group leader's values (lanes of groups that went to a peer buffer above
  // have returned, so the mask is the group, not every active lane)
  base = __shfl_sync(grp, base, leader);
  c0 = __shfl_sync(grp, c0, leader);
  c1 = __shfl_sync(grp, c1, leader);
  const unsigned long long pos = base + rank;
  const uint32_t c = ((pos >> pl.c_shift) == (base >> pl.c_shift)) ? c0 : c1;
  pl.slots[((uint64_t)c << pl.c_shift) | (pos & cmask)] = rec;
}

__device__ __forceinline__ unsigned long long warp_sum(unsigned long long x) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(kFull, x, o);
  return x;
}

// ---- walk record formats (16 B, D5; current_vertex + walked_steps, plus the walk id)
//   V: {row, v, t, 0}                                   (t < 2^31)
//   O: {row, off lo32, t | off hi8 << 23 | 1 << 31, deg}  (t < 2^23, off < 2^40)
// O carries the offset and degree of the current vertex instead of the vertex itself: with the
// augmented layouts the last gather of a walk that leaves a partition already returned them, so its
// next visit starts with the neighbour gather instead of a dependent random row_ptr read (DESIGN.md §7,
// "P > 1"). Only walks appended to a LOCAL bucket by an update kernel take O (v is then not needed: a
// visit's next vertex comes from the gather); records for other ranks and every record written by
// k_init / k_insert_records are V (a receiver needs v to find the partition).
__device__ __forceinline__ bool rec_is_o(const uint4& r) { return (r.z >> 31) != 0; }
__device__ __forceinline__ uint4 rec_make_o(uint32_t row, uint32_t t, unsigned long long off, uint32_t deg) {
  return make_uint4(row, (uint32_t)off, t | ((uint32_t)(off >> 32) << 23) | 0x80000000u, deg);
}
__device__ __forceinline__ bool rec_fits_o(uint32_t t, unsigned long long off) {
  return t < (1u << 23) && (off >> 40) == 0;
}
// Decode a record loaded from a bucket into the working state (rec.z = t; rec.y = v for V records, kEmpty
// for O records); returns true and the current vertex's offset and degree for an O record.
__device__ __forceinline__ bool rec_decode(uint4& r, unsigned long long& off, uint32_t& deg) {
  if (!rec_is_o(r)) return false;
  off = (unsigned long long)r.y | ((unsigned long long)((r.z >> 23) & 0xFFu) << 32);
  deg = r.w;
  r.z &= 0x7FFFFFu;
  r.y = kEmpty;
  r.w = 0;
  return true;
}

// Retire after the last CTA of a launch over bucket k: free the chunks wholly below the consumed
// position `tail` (back onto the free stack, ring slots emptied) and advance head[k] (a6).
__device__ void last_cta_retire(const Params& p, int k, unsigned long long head, unsigned long long tail) {
  __shared__ bool s_last;
  __syncthreads();
  if (threadIdx.x == 0) {
    // peer-memory appends (walks for other ranks) and remote path entries performed before the grid ends
    if (p.peer.recv || p.sys_fence) __threadfence_system();
    else __threadfence();
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
      if (c >= pl.num_chunks) continue;  // a direct-start bucket's virtual chunk (or the trash chunk)
      const int idx = atomicAdd(pl.free_top, 1);
      if (idx >= 0) pl.free_list[idx] = c;
    }
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    if (k >= 0) {
      pl.head[(uint64_t)k * pl.hs] = tail;
      pl.claim[(uint64_t)k * pl.hs] = tail;  // refill claims may have run past the snapshot
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

// Bucket of partition q seen from this rank: q itself when owned, else the send bucket of its owner.
__device__ __forceinline__ uint32_t bucket_of(const Params& p, uint32_t q) {
  if (q >= p.own.own_lo && q < p.own.own_hi) return q;
  return p.wk.P + p.own.owner[q];
}

// ------------------------------------------------------------------------------------------ a2
// Walk init: path[w][0] and insertion into the start partition's bucket. With range ownership
// (world > 1) every rank sees every start and keeps the walks whose start partition it owns.
__global__ void __launch_bounds__(256) k_init(Params p, const uint32_t* __restrict__ starts, uint64_t W,
                                              uint64_t first_row) {
  extern __shared__ uint32_t s_bounds[];
  const Walk& wk = p.wk;
  const uint32_t* B = stage_bounds(wk, s_bounds);
  const uint32_t lane = threadIdx.x & 31u;
  const uint64_t nwarps = (uint64_t)gridDim.x * (blockDim.x >> 5);
  for (uint64_t base = ((uint64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) * 32; base < W;
       base += nwarps * 32) {
    const uint64_t j = base + lane;  // walk j of this admission = row first_row + j
    const uint64_t i = first_row + j;
    bool have = j < W;
    uint4 rec = make_uint4(0, 0, 0, 0);
    uint32_t dest = 0;
    if (have) {
      const uint32_t v = starts[j];
      dest = find_partition(B, wk.P, v);
      have = dest >= p.own.own_lo && dest < p.own.own_hi;
      if (have) {
        // path[w][0]: with buffered path stores (path_mode 0) the update kernel writes the walk's first
        // sector, entry 0 included, on the walk's first visit, so only the per-step mode stores it here
        if (wk.path_mode == 1) wk.paths[i * wk.pitch] = v;
        if (wk.visits16) {  // the start is the walk's first visit (VIS 3: the counter by degree)
          const uint32_t dg = (uint32_t)(__ldg(wk.row_ptr + v + 1) - __ldg(wk.row_ptr + v));
          if (dg >= wk.hub_deg) atomicAdd(wk.visits32 + v, 1u);
          else atomicAdd(wk.visits16 + (v >> 1), (v & 1u) ? 0x10000u : 1u);
        } else if (wk.visits32) atomicAdd(wk.visits32 + v, 1u);
        else if (wk.visits) atomicAdd(wk.visits + v, 1ull);
        rec = make_uint4((uint32_t)i, v, 0u, 0u);
      }
    }
    insert_warp(p, have, dest, rec);
  }
  last_cta_retire(p, -1, 0, 0);
}

// a9 receive side: records that arrived from other ranks go into the buckets of their (owned)
// partitions with the same warp-aggregated insertion.
__global__ void __launch_bounds__(256) k_insert_records(Params p, const uint4* __restrict__ recs, uint64_t count,
                                                        const unsigned long long* __restrict__ dcount) {
  extern __shared__ uint32_t s_bounds[];
  // fused superstep: the count is read on the device (no host round trip); a cursor past the buffer
  // (an overflow, flagged by the sender and reported by its lt_run) is clamped to what was stored
  if (dcount) count = (*dcount < p.peer.cap) ? *dcount : p.peer.cap;
  const Walk& wk = p.wk;
  const uint32_t* B = stage_bounds(wk, s_bounds);
  const uint32_t lane = threadIdx.x & 31u;
  const uint64_t nwarps = (uint64_t)gridDim.x * (blockDim.x >> 5);
  for (uint64_t base = ((uint64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) * 32; base < count;
       base += nwarps * 32) {
    const uint64_t i = base + lane;
    const bool have = i < count;
    uint4 rec = make_uint4(0, 0, 0, 0);
    uint32_t dest = 0;
    if (have) {
      rec = recs[i];
      dest = bucket_of(p, find_partition(B, wk.P, rec.y));
    }
    insert_warp(p, have, dest, rec);
  }
  last_cta_retire(p, -1, 0, 0);
}

// a9 send side: copy send bucket `bucket` ([head, cursor), read at launch) contiguously to `out`
// and retire its chunks.
__global__ void __launch_bounds__(256) k_pack(Params p, uint32_t bucket, uint4* __restrict__ out) {
  const Pool& pl = p.pool;
  const unsigned long long head = pl.head[(uint64_t)bucket * pl.hs], tail = pl.cursor[(uint64_t)bucket * pl.hs];
  const uint32_t* ring_b = pl.ring + (uint64_t)bucket * pl.ring_len;
  for (unsigned long long pos = head + (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; pos < tail;
       pos += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t c = ring_b[(pos >> pl.c_shift) % pl.ring_len];
    out[pos - head] = pl.slots[((uint64_t)c << pl.c_shift) | (pos & (pl.C - 1))];
  }
  last_cta_retire(p, (int)bucket, head, tail);
}

// Gather loads. GM selects L2 cache hints:
//   0: plain ld.global.nc everywhere
//   3: the per-step neighbour gather (col / adj) with an L2 evict_first policy (those lines are
//      never reused) and the L2::64B prefetch-size hint (halves the DRAM bytes of each miss); the
//      row_ptr gathers keep the default policy so the hot vertices' offsets stay in L2.
struct Policies {
  uint64_t first;
};
__device__ __forceinline__ Policies make_policies() {
  Policies p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p.first));
  return p;
}

// Path-entry stores: every path sector is written once and never read back
// by the walk; LT_PATH_HINT=1 sends it to L2 with the evict_first policy so it does not push out the
// lines the step re-reads (row_ptr of hot vertices, bucket tails, visit counters). Off by default.
#ifndef LT_PATH_HINT
#define LT_PATH_HINT 0  // measured: evict_first path stores cost DeepWalk 2 % (67.4 vs 66.0 ms), gain PageRank < 1 %
#endif
__device__ __forceinline__ void st_sector(uint32_t* dst, const uint32_t* v, const Policies& pol) {
#if LT_PATH_HINT
  asm volatile("st.global.L2::cache_hint.v4.u32 [%0], {%1, %2, %3, %4}, %5;"
               :: "l"(dst), "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "l"(pol.first) : "memory");
  asm volatile("st.global.L2::cache_hint.v4.u32 [%0], {%1, %2, %3, %4}, %5;"
               :: "l"(dst + 4), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]), "l"(pol.first) : "memory");
#else
  uint4* d = reinterpret_cast<uint4*>(dst);
  d[0] = make_uint4(v[0], v[1], v[2], v[3]);
  d[1] = make_uint4(v[4], v[5], v[6], v[7]);
#endif
}
// The per-step row_ptr pair of the CSR layout (LT_RP_HINT=1: L2 evict_last, so the offsets of hot
// vertices survive the streaming col gathers and path stores).
#ifndef LT_RP_HINT
#define LT_RP_HINT 0
#endif
__device__ __forceinline__ unsigned long long ld_rp(const unsigned long long* p) {
#if LT_RP_HINT == 1
  unsigned long long v;
  asm volatile("{\n\t.reg .b64 pol;\n\tcreatepolicy.fractional.L2::evict_last.b64 pol, 1.0;\n\t"
               "ld.global.nc.L2::cache_hint.u64 %0, [%1], pol;\n\t}" : "=l"(v) : "l"(p));
  return v;
#elif LT_RP_HINT == 2  // 64-B DRAM fills instead of 128-B lines on a miss
  unsigned long long v;
  asm volatile("ld.global.nc.L2::64B.u64 %0, [%1];" : "=l"(v) : "l"(p));
  return v;
#elif LT_RP_HINT == 3
  unsigned long long v;
  asm volatile("{\n\t.reg .b64 pol;\n\tcreatepolicy.fractional.L2::evict_last.b64 pol, 1.0;\n\t"
               "ld.global.nc.L2::cache_hint.L2::64B.u64 %0, [%1], pol;\n\t}" : "=l"(v) : "l"(p));
  return v;
#else
  return __ldg(p);
#endif
}

// A visit's (or a restart's) offset and degree from row_ptr with augmented layouts: a random vertex, so
// with GM != 0 each read fills a 64-B DRAM block (L2::64B) instead of a 128-B line (PageRank restarts are
// 15 % of its steps).
#ifndef LT_RP64
#define LT_RP64 1
#endif
template <int GM>
__device__ __forceinline__ void rp_pair(const unsigned long long* p, unsigned long long& off, uint32_t& d) {
  if (GM == 0 || !LT_RP64) {
    off = __ldg(p);
    d = (uint32_t)(__ldg(p + 1) - off);
    return;
  }
  unsigned long long a, b;
  asm volatile("ld.global.nc.L2::64B.u64 %0, [%1];" : "=l"(a) : "l"(p));
  asm volatile("ld.global.nc.L2::64B.u64 %0, [%1];" : "=l"(b) : "l"(p + 1));
  off = a;
  d = (uint32_t)(b - a);
}

// VIS 4: a vertex's offset, degree and counter slot from the per-vertex table vinfo = {off lo32, off hi8 |
// slot << 8, deg, 0} (one 16-B read where rp_pair would read row_ptr twice, and the slot lets a restart or a
// start count in the slot counters instead of a random per-vertex counter).
#ifndef LT_VINFO
#define LT_VINFO 1
#endif
template <int VIS, int GM>
__device__ __forceinline__ void vert_info(const Walk& wk, uint32_t v, unsigned long long& off, uint32_t& d,
                                          uint32_t& slot) {
  if (VIS == 4 && LT_VINFO) {
    uint4 q;
    asm volatile("ld.global.nc.L2::64B.v4.u32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(q.x), "=r"(q.y), "=r"(q.z), "=r"(q.w) : "l"(wk.vinfo + v));
    off = (unsigned long long)q.x | ((unsigned long long)(q.y & 0xFFu) << 32);
    d = q.z;
    slot = q.y >> 8;
    return;
  }
  rp_pair<GM>(wk.row_ptr + v, off, d);
  slot = 0;
}

template <int GM>
__device__ __forceinline__ uint32_t ld_col(const uint32_t* p, const Policies& pol) {
  if (GM == 0) return __ldg(p);
  uint32_t v;
  asm volatile("ld.global.nc.L2::cache_hint.L2::64B.u32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol.first));
  return v;
}
template <int GM>
__device__ __forceinline__ uint4 ld_adj(const uint4* p, const Policies& pol) {
  if (GM == 0) return __ldg(p);
  uint4 v;
  asm volatile("ld.global.nc.L2::cache_hint.L2::64B.v4.u32 {%0, %1, %2, %3}, [%4], %5;"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
               : "l"(p), "l"(pol.first));
  return v;
}

// The first step of a walk (t = 0) gathers from its start vertex's adjacency with an L2 evict_last policy:
// when many walks share a start (PPR: every walk starts at the source) those lines are re-read by every
// walk, unlike the entries of later steps (evict_first, never reused). LT_FIRST_KEEP=0 turns it off.
#ifndef LT_FIRST_KEEP
#define LT_FIRST_KEEP 1
#endif
template <int GM>
__device__ __forceinline__ uint4 ld_adj_step(const uint4* p, const Policies& pol, bool first) {
  if (GM != 0 && LT_FIRST_KEEP && first) {
    uint4 v;
    asm volatile("{\n\t.reg .b64 pk;\n\tcreatepolicy.fractional.L2::evict_last.b64 pk, 1.0;\n\t"
                 "ld.global.nc.L2::cache_hint.L2::64B.v4.u32 {%0, %1, %2, %3}, [%4], pk;\n\t}"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
    return v;
  }
  return ld_adj<GM>(p, pol);
}

// Compact augmented adjacency (LAY 2): entry j is 12 bytes = 3 words {u, off lo32, off hi8 | deg << 8}
// (row_ptr[u] < 2^40, deg(u) < 2^24). Two aligned 8-B loads cover the entry wherever it starts (byte
// 12j is 8-aligned for even j, 4 past an 8-B boundary for odd j); they fall in one 64-B block unless the
// entry itself straddles one (2 of every 16 entries), so a step is still ONE random DRAM access.
struct Adj { uint32_t u, deg; unsigned long long off; };
#ifndef LT_ADJ12_LOAD
#define LT_ADJ12_LOAD 0  // 0: two 8-B loads; 1: three 4-B loads; 2: 16-B load + a second one when needed
#endif
#ifndef LT_ADJ12_POL
#define LT_ADJ12_POL 0   // 0: evict_first + L2::64B (GM 3); 1: L2::64B only
#endif
template <int GM>
__device__ __forceinline__ uint2 ld2_hint(const uint2* q, const Policies& pol) {
  uint2 v;
  if (GM == 0) return __ldg(q);
#if LT_ADJ12_POL == 0
  asm volatile("ld.global.nc.L2::cache_hint.L2::64B.v2.u32 {%0, %1}, [%2], %3;" : "=r"(v.x), "=r"(v.y) : "l"(q), "l"(pol.first));
#else
  asm volatile("ld.global.nc.L2::64B.v2.u32 {%0, %1}, [%2];" : "=r"(v.x), "=r"(v.y) : "l"(q));
#endif
  return v;
}
template <int GM>
__device__ __forceinline__ uint32_t ld1_hint(const uint32_t* q, const Policies& pol) {
  uint32_t v;
  if (GM == 0) return __ldg(q);
  asm volatile("ld.global.nc.L2::cache_hint.L2::64B.u32 %0, [%1], %2;" : "=r"(v) : "l"(q), "l"(pol.first));
  return v;
}
template <int GM>
__device__ __forceinline__ Adj ld_adj12(const uint32_t* a12, unsigned long long j, const Policies& pol) {
  const unsigned long long w = 3 * j;  // word index of the entry
  uint32_t w0, w1, w2;
#if LT_ADJ12_LOAD == 1
  w0 = ld1_hint<GM>(a12 + w, pol);
  w1 = ld1_hint<GM>(a12 + w + 1, pol);
  w2 = ld1_hint<GM>(a12 + w + 2, pol);
#elif LT_ADJ12_LOAD == 2
  const uint4* q4 = reinterpret_cast<const uint4*>(a12 + (w & ~3ull));
  const uint4 A = ld_adj<GM>(q4, pol);
  const uint32_t r = (uint32_t)(w & 3ull);
  uint4 B = make_uint4(0, 0, 0, 0);
  if (r >= 2) B = ld_adj<GM>(q4 + 1, pol);
  w0 = r == 0 ? A.x : r == 1 ? A.y : r == 2 ? A.z : A.w;
  w1 = r == 0 ? A.y : r == 1 ? A.z : r == 2 ? A.w : B.x;
  w2 = r == 0 ? A.z : r == 1 ? A.w : r == 2 ? B.x : B.y;
#else
  const uint2* q = reinterpret_cast<const uint2*>(a12 + (w & ~1ull));
  const uint2 lo = ld2_hint<GM>(q, pol), hi = ld2_hint<GM>(q + 1, pol);
  const bool odd = (w & 1ull) != 0;
  w0 = odd ? lo.y : lo.x;
  w1 = odd ? hi.x : lo.y;
  w2 = odd ? hi.y : hi.x;
#endif
  Adj e;
  e.u = w0;
  e.deg = w2 >> 8;
  e.off = (unsigned long long)w1 | ((unsigned long long)(w2 & 0xFFu) << 32);
  return e;
}

// ------------------------------------------------------------------------------- a3 + a4 + a5
// ILP walks per lane: a warp takes 32*ILP consecutive records; each lane advances its ILP walks in
// lockstep so their dependent gathers are in flight together (memory-level parallelism is what
// bounds this kernel: the measured random-access rate of the HBM).
// LAY selects the graph layout the step gathers from:
//   0 (CSR): per step row_ptr[v], row_ptr[v+1] (one line) then col[off + i] (one line);
//   1 (ADJ): per step ONE 16-B gather adj[off + i] = {u, deg(u), row_ptr[u]} that carries the next
//            vertex's degree and offset, so only a visit's first step reads row_ptr.
// Offsets are global CSR positions; col / adj hold the entries from wk.ebase on (an out-of-core
// block's slice, or the owned slice with range ownership), so every gather subtracts ebase.
#ifndef LT_UPD_MINB
#define LT_UPD_MINB 4  // resident 256-thread blocks per SM the batch kernel's registers are cut for (ILP 1)
#endif
template <int ILP> struct MinBlocks { static constexpr int v = LT_UPD_MINB; };
template <> struct MinBlocks<2> { static constexpr int v = 3; };
template <> struct MinBlocks<4> { static constexpr int v = 2; };

// VIS: fused per-vertex visit counting (lt_config.visit_counts) compiled out (0), with u64 counters
// (1), or with u32 counters (2, while every count fits): the default kernels carry no trace of it.
// The add is a fire-and-forget RED to the vertex's counter, resolved in L2.
// The counters carry an L2 evict_last policy: they are the only lines of the step that are re-read
// at random (visits are degree-skewed, so the hot counters stay resident).
#ifndef LT_VIS_HINT
#define LT_VIS_HINT 1
#endif
// VIS 3 (round 2): two 16-bit counters per 32-bit word (vertex v in half v & 1 of word v >> 1; the
// n/2-word array is half the size of the u32 one, so far more of it stays in L2), except for hub vertices
// (degree >= wk.hub_deg, whose expected count is too large for 16 bits), which count in the u32 array.
// The degree of the visited vertex comes with the step (the augmented entry), so choosing costs no load.
// A 16-bit half that wraps is detected exactly at the end of lt_run (the sum of all counts falls short of
// the number of path entries) and the counts are then recomputed from the paths.
// VIS 4 (round 2, the ADJ layout): the hottest vertices' counters packed densely by degree rank. The ADJ
// entry of a step carries the visited vertex's *slot* (its rank by degree + 1, for the 2^24 - 1 highest
// degrees; 0 for the rest) in the spare bits of its offset word, so a visit through an edge counts in
// vhot[slot] — a 64-MB array whose hot prefix (the vertices most visits go to) stays in L2 — and every
// other visit (starts, restarts, unslotted vertices) in the per-vertex u32 array visits32. The result is
// their sum per vertex (k_widen_slots); every count is < 2^32 (W * stride < 2^32), so nothing can wrap.
template <int VIS>
__device__ __forceinline__ void count_visit(const Walk& wk, uint32_t v, uint32_t deg, uint64_t pol_last,
                                            uint32_t slot = 0) {
  if (VIS == 4) {
    if (slot)
      asm volatile("red.relaxed.gpu.global.add.L2::cache_hint.u32 [%0], 1, %1;" :: "l"(wk.vhot + hot_index(slot)), "l"(pol_last)
                   : "memory");
    else
      asm volatile("red.relaxed.gpu.global.add.u32 [%0], 1;" :: "l"(wk.visits32 + v) : "memory");
    return;
  }
  (void)slot;
  if (VIS == 3) {
    if (deg >= wk.hub_deg)
      asm volatile("red.relaxed.gpu.global.add.L2::cache_hint.u32 [%0], 1, %1;" :: "l"(wk.visits32 + v), "l"(pol_last)
                   : "memory");
    else
      asm volatile("red.relaxed.gpu.global.add.L2::cache_hint.u32 [%0], %1, %2;" :: "l"(wk.visits16 + (v >> 1)),
                   "r"((v & 1u) ? 0x10000u : 1u), "l"(pol_last) : "memory");
    return;
  }
  (void)deg;
#if LT_VIS_HINT
  if (VIS == 1)
    asm volatile("red.relaxed.gpu.global.add.L2::cache_hint.u64 [%0], 1, %1;" :: "l"(wk.visits + v), "l"(pol_last)
                 : "memory");
  if (VIS == 2)
    asm volatile("red.relaxed.gpu.global.add.L2::cache_hint.u32 [%0], 1, %1;" :: "l"(wk.visits32 + v), "l"(pol_last)
                 : "memory");
#else
  (void)pol_last;
  if (VIS == 1) atomicAdd(wk.visits + v, 1ull);
  if (VIS == 2) atomicAdd(wk.visits32 + v, 1u);
#endif
}
__device__ __forceinline__ uint64_t make_evict_last() {
  uint64_t p = 0;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}

template <int APP, int GM, int ILP, int LAY, int VIS>
__global__ void __launch_bounds__(256, MinBlocks<ILP>::v) k_update(Params p, uint32_t k) {
  extern __shared__ uint32_t s_bounds[];
  const Walk& wk = p.wk;
  const Pool& pl = p.pool;
  const uint32_t* B = stage_bounds(wk, s_bounds);
  const unsigned long long head = pl.head[(uint64_t)k * pl.hs];
  // no appends to bucket k during its own launch; a spill-limited launch stops at tail_cap (the first
  // position of the bucket's first chunk still in host memory)
  const unsigned long long cur_k = pl.cursor[(uint64_t)k * pl.hs];
  const unsigned long long tail = cur_k < p.tail_cap ? cur_k : p.tail_cap;
  const uint32_t lo = wk.bounds[k];
  const uint32_t span = wk.bounds[k + 1] - lo;
  const uint32_t lane = threadIdx.x & 31u;
  const uint64_t nwarps = (uint64_t)gridDim.x * (blockDim.x >> 5);
  const uint32_t* ring_k = pl.ring + (uint64_t)k * pl.ring_len;
  const Policies pol = make_policies();
  const uint64_t pol_last = VIS ? make_evict_last() : 0;
  unsigned long long my_steps = 0, my_trunc = 0;
  __shared__ unsigned long long s_sent;
  if (threadIdx.x == 0) s_sent = 0;
  __syncthreads();

  for (unsigned long long base = head + ((uint64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) * (32 * ILP);
       base < tail; base += nwarps * (32 * ILP)) {
    uint4 rec[ILP];  // .x = row, .y = current vertex v, .z = walked steps t
    bool alive[ILP], left[ILP], trunc[ILP];
    uint32_t* prow[ILP];
    // Path entries are buffered per walk in a shift register (pb[s][7] = newest, entry t) and written
    // as full 32-B sectors (two 16-B stores) whenever entry t closes a sector (t % 8 == 7); `nb`
    // counts the buffered entries not yet in memory. The visit's first vertex (entry t0, already in
    // memory) seeds the buffer so a sector that starts at t0 can still be written whole.
    uint32_t pb[ILP][8];
    uint32_t nb[ILP];
    unsigned long long off[ILP];
    uint32_t d[ILP];
    bool kn[ILP];  // off / d belong to the current vertex (augmented layouts; false after a restart that left)
#pragma unroll
    for (int s = 0; s < ILP; ++s) {
      const unsigned long long pos = base + s * 32 + lane;
      alive[s] = pos < tail;
      left[s] = false;
      trunc[s] = false;
      rec[s] = make_uint4(0, 0, 0, 0);
      if (alive[s]) {
        const uint32_t c = ring_k[(pos >> pl.c_shift) % pl.ring_len];
        rec[s] = __ldcs(pl.slots + (((uint64_t)c << pl.c_shift) | (pos & (pl.C - 1))));
      }
      off[s] = 0;
      d[s] = 0;
      const bool o = LAY != 0 && rec_decode(rec[s], off[s], d[s]);
      prow[s] = wk.paths + (uint64_t)rec[s].x * wk.pitch;
      kn[s] = LAY != 0;
#pragma unroll
      for (int q = 0; q < 8; ++q) pb[s][q] = 0;
      pb[s][7] = rec[s].y;
      // entry t0 opens its sector: rewrite it too (an O record does not carry v: its sector is then
      // written from t0 + 1 on, a partial sector)
      nb[s] = (alive[s] && !o && (rec[s].z & 7u) == 0) ? 1u : 0u;
      if (LAY != 0 && alive[s] && !o) {  // the visit's first vertex: its offset and degree from row_ptr
        rp_pair<GM>(wk.row_ptr + rec[s].y, off[s], d[s]);
      }
    }
    for (;;) {
      bool any = false;
#pragma unroll
      for (int s = 0; s < ILP; ++s) {
        if (alive[s]) {
          if (APP != 1) {  // DeepWalk and PageRank: fixed length l
            if (rec[s].z == wk.length) alive[s] = false;
          } else if (rec[s].z == wk.lmax) {
            trunc[s] = true;
            alive[s] = false;
          }
        }
        any |= alive[s];
      }
      if (!any) break;
      if (LAY == 0) {
#pragma unroll
        for (int s = 0; s < ILP; ++s) {  // issue every row_ptr gather first
          if (alive[s]) {
            // the loaded graph may be one partition's slice (out-of-core pool block or a zero-copy
            // host view): row_ptr is indexed from vbase and col from ebase
            const unsigned long long* rp = wk.row_ptr + (rec[s].y - wk.vbase);
            const unsigned long long r0 = ld_rp(rp), r1 = ld_rp(rp + 1);
            off[s] = r0 - wk.ebase;
            d[s] = (uint32_t)(r1 - r0);
          }
        }
      }
      uint4 b[ILP];
#pragma unroll
      for (int s = 0; s < ILP; ++s) {  // Philox overlaps the gather latency (it needs only w and t)
        const uint64_t wid = wk.first_walk_id + rec[s].x;
        b[s] = philox10(make_uint4(rec[s].z, 0u, (uint32_t)wid, (uint32_t)(wid >> 32)), wk.seed_lo, wk.seed_hi);
      }
      uint32_t nv[ILP], sl[ILP];
#pragma unroll
      for (int s = 0; s < ILP; ++s) {
        nv[s] = 0;
        sl[s] = 0;
        if (APP == 1 && alive[s] && b[s].x < wk.T) alive[s] = false;  // terminate before moving
        const bool restart = APP == 2 && alive[s] && b[s].x < wk.T;    // PageRank: jump to a uniform vertex
        if (alive[s] && !restart && d[s] == 0) alive[s] = false;        // dead end
        if (alive[s]) {
          const uint32_t dd = restart ? wk.n : d[s];  // the draw ranges over [0, n) on a restart
          const uint64_t m = (uint64_t)b[s].y * dd;
          const uint64_t wid = wk.first_walk_id + rec[s].x;
          const uint32_t idx = ((uint32_t)m < dd)
                                   ? lemire_slow(dd, b[s], rec[s].z, (uint32_t)wid, (uint32_t)(wid >> 32),
                                                 wk.seed_lo, wk.seed_hi)
                                   : (uint32_t)(m >> 32);
          if (restart) {
            nv[s] = idx;
            kn[s] = LAY != 0 && (idx - lo < span || VIS >= 3);
            if (kn[s]) {  // staying (or VIS 3 / 4: its degree / slot picks the counter): its offset and degree
              vert_info<VIS, GM>(wk, idx, off[s], d[s], sl[s]);
            }
          } else if (LAY == 0) {
            nv[s] = ld_col<GM>(wk.col + off[s] + idx, pol);
          } else if (LAY == 1) {
            const uint4 e = ld_adj_step<GM>(wk.adj + (off[s] - wk.ebase) + idx, pol, rec[s].z == 0);
            nv[s] = e.x;
            d[s] = e.y;
            off[s] = (unsigned long long)e.z | ((unsigned long long)(e.w & 0xFFu) << 32);
            sl[s] = e.w >> 8;
          } else {
            const Adj e = ld_adj12<GM>(wk.adj12, off[s] - wk.ebase + idx, pol);
            nv[s] = e.u;
            d[s] = e.deg;
            off[s] = e.off;
          }
        }
      }
#pragma unroll
      for (int s = 0; s < ILP; ++s) {
        if (alive[s]) {
          rec[s].y = nv[s];
          rec[s].z += 1;
          count_visit<VIS>(wk, nv[s], d[s], pol_last, sl[s]);
          const uint32_t t = rec[s].z;
          if (wk.path_mode == 0) {
#pragma unroll
            for (int q = 0; q < 7; ++q) pb[s][q] = pb[s][q + 1];
            pb[s][7] = nv[s];
            nb[s] += 1;
            if ((t & 7u) == 7u) {  // entry t closes sector [t-7, t]
              if (nb[s] == 8) {
                st_sector(prow[s] + (t - 7), pb[s], pol);
              } else {
#pragma unroll
                for (int q = 0; q < 8; ++q)
                  if ((uint32_t)q < nb[s]) prow[s][t - q] = pb[s][7 - q];
              }
              nb[s] = 0;
            }
          } else if (wk.path_mode == 1) {
            prow[s][t] = nv[s];
          }
          if (nv[s] - lo >= span) {
            left[s] = true;
            alive[s] = false;
          }
        }
      }
    }
#pragma unroll
    for (int s = 0; s < ILP; ++s) {  // flush the entries of an unfinished sector
      if (wk.path_mode == 0) {
        const uint32_t t = rec[s].z;
#pragma unroll
        for (int q = 0; q < 8; ++q)
          if ((uint32_t)q < nb[s]) prow[s][t - q] = pb[s][7 - q];
      }
    }
#pragma unroll
    for (int s = 0; s < ILP; ++s) {
      const bool had = base + s * 32 + lane < tail;
      uint32_t dest = 0;
      if (had) {
        if (left[s]) {
          dest = bucket_of(p, find_partition(B, wk.P, rec[s].y));
          if (LAY != 0 && kn[s] && dest < wk.P && rec_fits_o(rec[s].z, off[s]))
            rec[s] = rec_make_o(rec[s].x, rec[s].z, off[s], d[s]);
        } else {
          wk.lengths[rec[s].x] = rec[s].z + 1;
          my_steps += rec[s].z;
          my_trunc += trunc[s] ? 1 : 0;
        }
      }
      insert_warp(p, had && left[s], dest, rec[s], &s_sent);
    }
  }
  my_steps = warp_sum(my_steps);
  my_trunc = warp_sum(my_trunc);
  if (lane == 0 && my_steps) atomicAdd(&p.ctr->steps, my_steps);
  if (lane == 0 && my_trunc) atomicAdd(&p.ctr->truncated, my_trunc);
  __syncthreads();
  if (threadIdx.x == 0 && s_sent) atomicAdd(&p.ctr->sent, s_sent);
  last_cta_retire(p, (int)k, head, tail);
}

// ------------------------------------------------------------------- a3 + a4 + a5, lane refill
// Same step, gathers and insertion as k_update, but a lane whose walk ended (terminated or left the
// partition) takes the next record of the bucket at once instead of idling until the warp's
// longest walk is done. Walk lengths inside a partition are geometric when P > 1 and for PPR, so
// without refill most lanes of a warp idle most of the time. A warp claims kRefill positions of the
// bucket at a time (one atomic per kRefill walks) and hands them to its idle lanes.
constexpr uint32_t kRefill = 64;
// Resident 256-thread blocks per SM the register budget is cut for. Measured on one B200 (DESIGN.md §8,
// profiles/r01_rf_minb_cmp.jsonl): 3 (up to 85 registers, no spills) is 2.6-3.0 % faster than 4 (64
// registers, 2 spilled) for DeepWalk cfg 4 and 1.2-1.7 % for PageRank; PPR's short walks want the 4th
// block (3: 1.3 % slower). LT_RF_MINB overrides all apps (experiments).
template <int APP> struct RfMinBlocks {
#ifdef LT_RF_MINB
  static constexpr int v = LT_RF_MINB;
#else
  static constexpr int v = APP == 1 ? 4 : 3;
#endif
};

// Sorted flush (LT_SORTED_FLUSH; lane refill with at most kSortBuckets buckets and C >= kStage): the warp's
// staged departures (up to kStage) are counted per destination in shared memory, ONE cursor atomic per
// destination reserves a contiguous run for all of them, and every record is stored at run base + its rank.
// Against 32-lane rounds (one atomic per (round, destination) group, runs of ~2 records at P = 16) this
// writes longer contiguous runs — whole 32-B sectors instead of partial ones the memory controller has to
// read-modify-write — and issues fewer cursor atomics.
#ifndef LT_SORTED_FLUSH
#define LT_SORTED_FLUSH 1
#endif
constexpr uint32_t kSortBuckets = 64;
#ifndef LT_STAGE_N
#define LT_STAGE_N 128
#endif
constexpr uint32_t kStage = LT_STAGE_N;  // staged departures per warp with the sorted flush (flushed at >= kStage - 32)
struct SortScratch {
  uint32_t hist[kSortBuckets];
  uint32_t c0[kSortBuckets], c1[kSortBuckets];
  unsigned long long base[kSortBuckets];
  uint32_t rank[kStage];
};

__device__ __forceinline__ void flush_sorted(const Params& p, const uint4* qr, const uint32_t* qd, uint32_t cnt,
                                             unsigned long long* sent_acc, SortScratch& ss) {
  const uint32_t lane = threadIdx.x & 31u;
  const Pool& pl = p.pool;
  const unsigned long long cmask = pl.C - 1;
  for (uint32_t d = lane; d < kSortBuckets; d += 32) ss.hist[d] = 0;
  __syncwarp();
  for (uint32_t i = lane; i < cnt; i += 32) ss.rank[i] = atomicAdd(&ss.hist[qd[i]], 1u);
  __syncwarp();
  for (uint32_t d = lane; d < kSortBuckets; d += 32) {  // one reservation per destination with departures
    const uint32_t n = ss.hist[d];
    if (!n) continue;
    if (p.peer.recv && d >= p.wk.P) {  // walks for rank q: a run in q's receive buffer (peer memory)
      const uint32_t slot = p.peer.epoch * (pl.nbuckets - p.wk.P) + (d - p.wk.P);
      const unsigned long long b = atomicAdd(p.peer.cursor[slot], (unsigned long long)n);
      if (b + n > p.peer.cap) atomicOr(&p.ctr->err, kErrPeer);
      atomicAdd(sent_acc, (unsigned long long)n);
      ss.base[d] = b;
      continue;
    }
    const unsigned long long b = atomicAdd(pl.cursor + (uint64_t)d * pl.hs, (unsigned long long)n);
    const unsigned long long ci0 = b >> pl.c_shift, ci1 = (b + n - 1) >> pl.c_shift;  // n <= C: two chunks
    uint32_t c1 = 0;
    if (ci1 != ci0) c1 = install_chunk(p, d, ci1);
    const uint32_t c0 = (b & cmask) == 0 ? install_chunk(p, d, ci0) : wait_chunk(p, d, ci0);
    ss.base[d] = b;
    ss.c0[d] = c0;
    ss.c1[d] = ci1 == ci0 ? c0 : c1;
  }
  __syncwarp();
  for (uint32_t i = lane; i < cnt; i += 32) {
    const uint32_t d = qd[i];
    const unsigned long long pos = ss.base[d] + ss.rank[i];
    if (p.peer.recv && d >= p.wk.P) {
      const uint32_t slot = p.peer.epoch * (pl.nbuckets - p.wk.P) + (d - p.wk.P);
      if (pos < p.peer.cap) p.peer.recv[slot][pos] = qr[i];
      continue;
    }
    const uint32_t c = ((pos >> pl.c_shift) == (ss.base[d] >> pl.c_shift)) ? ss.c0[d] : ss.c1[d];
    pl.slots[((uint64_t)c << pl.c_shift) | (pos & cmask)] = qr[i];
  }
  __syncwarp();
}

#ifndef LT_PAD_SECTOR
#define LT_PAD_SECTOR 1
#endif

// Insert `cnt` (<= 64) staged walks, 32 lanes per round (warp-collective).
__device__ __forceinline__ void flush_staged(const Params& p, const uint4* qr, const uint32_t* qd, uint32_t cnt,
                                             unsigned long long* sent_acc) {
  const uint32_t lane = threadIdx.x & 31u;
  for (uint32_t r = 0; r < cnt; r += 32) {
    const bool act = r + lane < cnt;
    insert_warp(p, act, act ? qd[r + lane] : 0u, act ? qr[r + lane] : make_uint4(0, 0, 0, 0), sent_acc);
  }
  __syncwarp();
}


// CONT (out-of-core, CSR layout only): resident-neighbour continuation (the
// paper's preemptive idea taken inside the kernel). Each lane carries its own graph
// view (row_ptr / col pointers pre-offset by the view's first vertex / first edge, and the range it
// covers); a walk that leaves the view for a partition whose block is in p.cont.table switches to that
// block's view and keeps stepping.
template <int APP, int GM, int LAY, int VIS, int CONT>
__global__ void __launch_bounds__(256, RfMinBlocks<APP>::v) k_update_rf(Params p, uint32_t k) {
  extern __shared__ uint32_t s_bounds[];
  const Walk& wk = p.wk;
  const Pool& pl = p.pool;
  const uint32_t* B = stage_bounds(wk, s_bounds);
  const unsigned long long head = pl.head[(uint64_t)k * pl.hs];
  const unsigned long long cur_k = pl.cursor[(uint64_t)k * pl.hs];
  const unsigned long long tail = cur_k < p.tail_cap ? cur_k : p.tail_cap;
  const uint32_t lo = wk.bounds[k];
  const uint32_t span = wk.bounds[k + 1] - lo;
  const uint32_t lane = threadIdx.x & 31u;
  const uint32_t* ring_k = pl.ring + (uint64_t)k * pl.ring_len;
  unsigned long long* claim = pl.claim + (uint64_t)k * pl.hs;
  const Policies pol = make_policies();
  const uint64_t pol_last = VIS ? make_evict_last() : 0;
  unsigned long long my_steps = 0, my_trunc = 0;
  __shared__ unsigned long long s_sent;
  if (threadIdx.x == 0) s_sent = 0;
  __syncthreads();

  bool has = false;
  uint4 rec = make_uint4(0, 0, 0, 0);  // .x = row, .y = v, .z = t
  uint32_t* prow = wk.paths;
  // the lane's graph view (CONT): row_ptr indexed by the global vertex, col by the global offset
  const unsigned long long* c_rp = wk.row_ptr - wk.vbase;
  const uint32_t* c_col = wk.col - wk.ebase;
  uint32_t c_lo = lo, c_span = span;
  uint32_t pb[8];
  uint32_t nb = 0;
  unsigned long long off = 0;
  uint32_t d = 0;
  bool kn = false;  // off / d belong to the current vertex (augmented layouts; false after a restart that left)
  unsigned long long q_cur = 0, q_end = 0;  // this warp's claimed, not yet handed out positions
  bool drained = false;
  __shared__ uint4 s_qr[8][kStage];     // per-warp staging of departing walks (records)
  __shared__ uint32_t s_qd[8][kStage];  // and their destination buckets
  __shared__ SortScratch s_ss[LT_SORTED_FLUSH ? 8 : 1];
  // the sorted flush when every bucket fits its histogram and a run of kStage records spans <= 2 chunks
  const bool sorted = LT_SORTED_FLUSH && pl.nbuckets <= kSortBuckets && pl.C >= kStage && p.insert_mode == 0;
  const uint32_t q_lim = sorted ? kStage - 32 : 32;
  const uint32_t wib = threadIdx.x >> 5;
  uint32_t q_cnt = 0;
#pragma unroll
  for (int q = 0; q < 8; ++q) pb[q] = 0;

  for (;;) {
    // ---- refill idle lanes from the warp's claimed range (claim kRefill more when it runs out)
    uint32_t need = __ballot_sync(kFull, !has);
    while (need && !drained) {
      if (q_cur >= q_end) {
        unsigned long long base = 0;
        if (lane == 0) base = atomicAdd(claim, (unsigned long long)kRefill);
        base = __shfl_sync(kFull, base, 0);
        q_cur = base;
        q_end = (base + kRefill < tail) ? base + kRefill : tail;
        if (q_cur >= tail) { drained = true; break; }
      }
      const uint32_t avail = (q_end - q_cur < 32ull) ? (uint32_t)(q_end - q_cur) : 32u;
      const uint32_t r = __popc(need & lanemask_lt());
      if (!has && r < avail) {
        const unsigned long long pos = q_cur + r;
        bool sv_count = false;
        if (pos < p.direct.count) {  // direct start: the new walk's record, built in registers (a2)
          rec = make_uint4((uint32_t)pos, __ldg(p.direct.starts + pos), 0u, 0u);
          if (wk.path_mode == 1) wk.paths[pos * wk.pitch] = rec.y;
          sv_count = true;  // the start is the walk's first visit (counted below, once its degree is known)
        } else {
          const uint32_t c = ring_k[(pos >> pl.c_shift) % pl.ring_len];
          rec = __ldcs(pl.slots + (((uint64_t)c << pl.c_shift) | (pos & (pl.C - 1))));
        }
        has = true;
        const bool o = LAY != 0 && rec_decode(rec, off, d);
        kn = LAY != 0;
        prow = wk.paths + (uint64_t)rec.x * wk.pitch;
        pb[7] = rec.y;
        nb = (!o && (rec.z & 7u) == 0) ? 1u : 0u;
        uint32_t s0 = 0;
        if (LAY != 0 && !o) vert_info<VIS, GM>(wk, rec.y, off, d, s0);
        if (sv_count) count_visit<VIS>(wk, rec.y, d, pol_last, s0);
        if (CONT) {  // a walk from the bucket starts in the launched partition's view
          c_rp = wk.row_ptr - wk.vbase;
          c_col = wk.col - wk.ebase;
          c_lo = lo;
          c_span = span;
        }
      }
      q_cur += (avail < (uint32_t)__popc(need)) ? avail : (uint32_t)__popc(need);
      need = __ballot_sync(kFull, !has);
    }
    if (!__any_sync(kFull, has)) break;
    // ---- one step of every lane that holds a walk
    bool done = false, left = false, trunc = false;
    if (has) {
      if (APP != 1 && rec.z == wk.length) {
        done = true;
      } else if (APP == 1 && rec.z == wk.lmax) {
        done = true;
        trunc = true;
      } else {
        if (LAY == 0) {
          if (CONT) {
            const unsigned long long* rp = c_rp + rec.y;
            off = ld_rp(rp);
            d = (uint32_t)(ld_rp(rp + 1) - off);
          } else {
            const unsigned long long* rp = wk.row_ptr + (rec.y - wk.vbase);
            const unsigned long long r0 = ld_rp(rp), r1 = ld_rp(rp + 1);
            off = r0 - wk.ebase;
            d = (uint32_t)(r1 - r0);
          }
        }
        const uint64_t wid = wk.first_walk_id + rec.x;
        const uint4 b = philox10(make_uint4(rec.z, 0u, (uint32_t)wid, (uint32_t)(wid >> 32)), wk.seed_lo, wk.seed_hi);
        const bool restart = APP == 2 && b.x < wk.T;  // PageRank: jump to a uniform vertex
        if ((APP == 1 && b.x < wk.T) || (d == 0 && !restart)) {
          done = true;
        } else {
          const uint32_t dd = restart ? wk.n : d;
          const uint64_t m = (uint64_t)b.y * dd;
          const uint32_t idx = ((uint32_t)m < dd) ? lemire_slow(dd, b, rec.z, (uint32_t)wid, (uint32_t)(wid >> 32),
                                                               wk.seed_lo, wk.seed_hi)
                                                  : (uint32_t)(m >> 32);
          uint32_t nv, sl = 0;
          if (restart) {
            nv = idx;
            kn = LAY != 0 && (idx - lo < span || VIS >= 3);
            if (kn) vert_info<VIS, GM>(wk, idx, off, d, sl);
          } else if (LAY == 0) {
            nv = ld_col<GM>((CONT ? c_col : wk.col) + off + idx, pol);
          } else if (LAY == 1) {
            const uint4 e = ld_adj_step<GM>(wk.adj + (off - wk.ebase) + idx, pol, rec.z == 0);
            nv = e.x;
            d = e.y;
            off = (unsigned long long)e.z | ((unsigned long long)(e.w & 0xFFu) << 32);
            sl = e.w >> 8;
          } else {
            const Adj e = ld_adj12<GM>(wk.adj12, off - wk.ebase + idx, pol);
            nv = e.u;
            d = e.deg;
            off = e.off;
          }
          rec.y = nv;
          rec.z += 1;
          count_visit<VIS>(wk, nv, d, pol_last, sl);
          const uint32_t t = rec.z;
          if (wk.path_mode == 0) {
#pragma unroll
            for (int q = 0; q < 7; ++q) pb[q] = pb[q + 1];
            pb[7] = nv;
            nb += 1;
            if ((t & 7u) == 7u) {
              if (nb == 8) {
                st_sector(prow + (t - 7), pb, pol);
              } else {
#pragma unroll
                for (int q = 0; q < 8; ++q)
                  if ((uint32_t)q < nb) prow[t - q] = pb[7 - q];
              }
              nb = 0;
            }
          } else if (wk.path_mode == 1) {
            prow[t] = nv;
          }
          if (CONT) {
            left = (nv - c_lo >= c_span);
            if (left) {  // into a resident partition: switch the view and keep stepping
              const uint32_t q = find_partition(B, wk.P, nv);
              const uint32_t blk = __ldg(p.cont.table + q);
              if (blk != kEmpty) {
                const char* base = p.cont.gpool + (uint64_t)blk * p.cont.block_bytes;
                const unsigned long long* rp = reinterpret_cast<const unsigned long long*>(base);
                c_lo = __ldg(wk.bounds + q);
                c_span = __ldg(wk.bounds + q + 1) - c_lo;
                c_rp = rp - c_lo;
                c_col = reinterpret_cast<const uint32_t*>(base + p.cont.rp_bytes) - __ldg(rp);
                left = false;
              }
            }
          } else {
            left = (nv - lo >= span);
          }
        }
      }
    }
    // ---- retire the walks that ended this step
    const bool ended = done || left;
    if (ended && wk.path_mode == 0) {
      const uint32_t t = rec.z;
      const uint32_t lo8 = t & 7u;  // the open sector holds entries [t - lo8, t]
      if (LT_PAD_SECTOR && done && nb > lo8) {
        // the walk ended and its open sector is wholly buffered: write the sector whole, the entries past
        // the end as the row padding (0xFFFFFFFF), instead of a partial sector the memory controller would
        // complete by read-modify-write (PPR: one per walk)
        uint32_t sec[8];
#pragma unroll
        for (int q = 0; q < 8; ++q) {  // sec[q] = pb[7 - lo8 + q] by selects (no dynamic register indexing)
          uint32_t v = kEmpty;
#pragma unroll
          for (int j = 0; j < 8; ++j)
            if ((uint32_t)j + lo8 == (uint32_t)q + 7u) v = pb[j];
          sec[q] = v;
        }
        st_sector(prow + (t - lo8), sec, pol);
      } else {
#pragma unroll
        for (int q = 0; q < 8; ++q)
          if ((uint32_t)q < nb) prow[t - q] = pb[7 - q];
      }
      nb = 0;
    }
    if (done) {
      wk.lengths[rec.x] = rec.z + 1;
      my_steps += rec.z;
      my_trunc += trunc ? 1 : 0;
    }
    // departing walks are staged per warp in shared memory and inserted 32-64 at a time, so the
    // destination cursors see one atomic per (flush round, destination) instead of one per
    // (step, destination): the warp-level form of the paper's local index
    const uint32_t lm = __ballot_sync(kFull, left);
    if (left) {
      const uint32_t slot = q_cnt + __popc(lm & lanemask_lt());
      const uint32_t dest = bucket_of(p, find_partition(B, wk.P, rec.y));
      s_qr[wib][slot] = (LAY != 0 && kn && dest < wk.P && rec_fits_o(rec.z, off)) ? rec_make_o(rec.x, rec.z, off, d) : rec;
      s_qd[wib][slot] = dest;
    }
    q_cnt += __popc(lm);
    if (q_cnt >= q_lim) {
      __syncwarp();
      if (sorted) flush_sorted(p, s_qr[wib], s_qd[wib], q_cnt, &s_sent, s_ss[LT_SORTED_FLUSH ? wib : 0]);
      else flush_staged(p, s_qr[wib], s_qd[wib], q_cnt, &s_sent);
      q_cnt = 0;
    }
    if (ended) has = false;
  }
  __syncwarp();
  if (sorted) flush_sorted(p, s_qr[wib], s_qd[wib], q_cnt, &s_sent, s_ss[LT_SORTED_FLUSH ? wib : 0]);
  else flush_staged(p, s_qr[wib], s_qd[wib], q_cnt, &s_sent);
  my_steps = warp_sum(my_steps);
  my_trunc = warp_sum(my_trunc);
  if (lane == 0 && my_steps) atomicAdd(&p.ctr->steps, my_steps);
  if (lane == 0 && my_trunc) atomicAdd(&p.ctr->truncated, my_trunc);
  __syncthreads();
  if (threadIdx.x == 0 && s_sent) atomicAdd(&p.ctr->sent, s_sent);
  last_cta_retire(p, (int)k, head, tail);
}


// ------------------------------------------------------------------------- walk spill (f3, a8)
// Eviction: block i copies chunk list[i] = (bucket, chunk index) into host slot
// list.slot[i] of the mapped host store (16-B stores over PCIe, 4 per thread in flight), marks the ring
// slot kSpilled and returns the device chunk to the free stack. Only full chunks strictly inside
// [head, cursor) of a bucket that is not being launched are listed, so no kernel reads or writes them while
// they live in host memory.
__global__ void __launch_bounds__(256) k_spill(Params p, SpillList list, uint4* __restrict__ store) {
  const Pool& pl = p.pool;
  __shared__ uint32_t s_c;
  uint32_t* slot = pl.ring + (uint64_t)list.bucket[blockIdx.x] * pl.ring_len + (list.chunk[blockIdx.x] % pl.ring_len);
  if (threadIdx.x == 0) s_c = *slot;
  __syncthreads();
  const uint32_t c = s_c;
  const uint4* src = pl.slots + ((uint64_t)c << pl.c_shift);
  uint4* dst = store + ((uint64_t)list.slot[blockIdx.x] << pl.c_shift);
  for (uint32_t i = threadIdx.x; i < pl.C; i += 4 * blockDim.x) {
    uint4 v[4];
#pragma unroll
    for (int u = 0; u < 4; ++u)
      if (i + u * blockDim.x < pl.C) v[u] = __ldcs(src + i + u * blockDim.x);
#pragma unroll
    for (int u = 0; u < 4; ++u)
      if (i + u * blockDim.x < pl.C) dst[i + u * blockDim.x] = v[u];
  }
  __threadfence_system();  // the host copy is complete before the chunk can be reused
  __syncthreads();
  if (threadIdx.x == 0) {
    *slot = kSpilled;
    const int idx = atomicAdd(pl.free_top, 1);
    pl.free_list[idx] = c;
  }
}

// Reload: block i pops a free device chunk, copies host slot list.slot[i] into it (reads over PCIe, 4 per
// thread in flight) and installs it in the ring slot of list[i] (which holds kSpilled).
__global__ void __launch_bounds__(256) k_reload(Params p, SpillList list, const uint4* __restrict__ store) {
  const Pool& pl = p.pool;
  __shared__ uint32_t s_c;
  uint32_t* slot = pl.ring + (uint64_t)list.bucket[blockIdx.x] * pl.ring_len + (list.chunk[blockIdx.x] % pl.ring_len);
  if (threadIdx.x == 0) {
    const int idx = atomicSub(pl.free_top, 1) - 1;
    uint32_t c = pl.num_chunks;  // trash chunk: flagged, cannot happen when the scheduler sized the reload
    if (idx >= 0) c = pl.free_list[idx];
    else atomicOr(&p.ctr->err, kErrOOM);
    if (*slot != kSpilled) atomicOr(&p.ctr->err, kErrRing);
    s_c = c;
  }
  __syncthreads();
  const uint32_t c = s_c;
  uint4* dst = pl.slots + ((uint64_t)c << pl.c_shift);
  const uint4* src = store + ((uint64_t)list.slot[blockIdx.x] << pl.c_shift);
  for (uint32_t i = threadIdx.x; i < pl.C; i += 4 * blockDim.x) {
    uint4 v[4];
#pragma unroll
    for (int u = 0; u < 4; ++u)
      if (i + u * blockDim.x < pl.C) v[u] = __ldcv(src + i + u * blockDim.x);  // not cached: host memory
#pragma unroll
    for (int u = 0; u < 4; ++u)
      if (i + u * blockDim.x < pl.C) dst[i + u * blockDim.x] = v[u];
  }
  __syncthreads();
  if (threadIdx.x == 0) *slot = c;
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
      uint32_t* prow = wk.paths + (base + j) * wk.pitch;
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
    out[i] = wk.paths[rows[r] * wk.pitch + t];
    if (t == 0) out_len[r] = wk.lengths[rows[r]];
  }
}

// Scheduler snapshot: head/cursor of every bucket, the counters and the free-stack top, written
// by the SMs straight into mapped pinned host memory. A cudaMemcpy would queue behind a large D2H
// on the same copy engine (lt_run_to_host's path copy-out) and serialise the pipeline.
// out_hc[b] = head of bucket b, out_hc[nb + b] = its cursor (compact, from the strided device blocks)
__global__ void k_snapshot(const unsigned long long* __restrict__ hc, uint64_t nb, uint32_t hs,
                           const Counters* __restrict__ ctr, const int* __restrict__ free_top,
                           volatile unsigned long long* out_hc, volatile Counters* out_ctr, volatile int* out_free) {
  for (uint64_t i = threadIdx.x; i < 2 * nb; i += blockDim.x) out_hc[i] = hc[(i % nb) * hs + i / nb];
  if (threadIdx.x == 0) {
    out_ctr->steps = ctr->steps;
    out_ctr->visits = ctr->visits;
    out_ctr->truncated = ctr->truncated;
    out_ctr->err = ctr->err;
    out_ctr->done_ctas = ctr->done_ctas;
    out_ctr->sent = ctr->sent;
    *out_free = *free_top;
  }
}

// Rows [0, n) of the pitched path matrix -> a dense n x stride buffer (one flat D2H afterwards), with
// the entries past each row's length written as 0xFFFFFFFF (the padding lt_run leaves undone).
__global__ void k_compact_rows(const uint32_t* __restrict__ paths, const uint32_t* __restrict__ lengths, uint64_t pitch,
                               uint64_t stride, uint64_t n, uint32_t* __restrict__ out) {
  const uint64_t total = n * stride;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t r = i / stride, t = i % stride;
    out[i] = t < __ldg(lengths + r) ? paths[r * pitch + t] : kEmpty;
  }
}

// ---- compact (ragged) path output: offsets = base + exclusive prefix sum of lengths, vertices packed.
// Three passes over tiles of kScanTile lengths: tile sums; one block scans the tile sums (and writes
// the total); each tile scans itself, writes its offsets and packs its rows (warp per row).
constexpr uint32_t kScanTile = 4096;  // 256 threads x 16 lengths

__global__ void __launch_bounds__(256) k_scan_tiles(const uint32_t* __restrict__ len, uint64_t n,
                                                   unsigned long long* __restrict__ tile_sum) {
  using Reduce = cub::BlockReduce<unsigned long long, 256>;
  __shared__ typename Reduce::TempStorage tmp;
  const uint64_t base = (uint64_t)blockIdx.x * kScanTile + threadIdx.x * 16;
  unsigned long long x = 0;
#pragma unroll
  for (int j = 0; j < 16; ++j)
    if (base + j < n) x += len[base + j];
  const unsigned long long t = Reduce(tmp).Sum(x);
  if (threadIdx.x == 0) tile_sum[blockIdx.x] = t;
}

__global__ void __launch_bounds__(1024) k_scan_tile_sums(unsigned long long* __restrict__ tile_sum, uint64_t ntiles,
                                                         unsigned long long* __restrict__ total) {
  using Scan = cub::BlockScan<unsigned long long, 1024>;
  __shared__ typename Scan::TempStorage tmp;
  __shared__ unsigned long long carry;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  for (uint64_t b = 0; b < ntiles; b += 1024) {
    const uint64_t i = b + threadIdx.x;
    unsigned long long x = i < ntiles ? tile_sum[i] : 0, agg = 0;
    Scan(tmp).ExclusiveSum(x, x, agg);
    if (i < ntiles) tile_sum[i] = x + carry;
    __syncthreads();
    if (threadIdx.x == 0) carry += agg;
    __syncthreads();
  }
  if (threadIdx.x == 0) *total = carry;
}

__global__ void __launch_bounds__(256) k_scan_apply(const uint32_t* __restrict__ len, uint64_t n,
                                                   const unsigned long long* __restrict__ tile_off,
                                                   unsigned long long base, unsigned long long* __restrict__ offsets,
                                                   const uint32_t* __restrict__ paths, uint64_t pitch,
                                                   uint32_t* __restrict__ vertices) {
  using Scan = cub::BlockScan<unsigned long long, 256>;
  __shared__ typename Scan::TempStorage tmp;
  __shared__ unsigned long long s_off[kScanTile];
  const uint64_t t0 = (uint64_t)blockIdx.x * kScanTile;
  const uint64_t mine = t0 + threadIdx.x * 16;
  unsigned long long v[16], x = 0;
#pragma unroll
  for (int j = 0; j < 16; ++j) {
    v[j] = (mine + j < n) ? len[mine + j] : 0;
    x += v[j];
  }
  Scan(tmp).ExclusiveSum(x, x);
  const unsigned long long tb = tile_off[blockIdx.x];  // local (0-based) offset of this tile
#pragma unroll
  for (int j = 0; j < 16; ++j) {
    s_off[threadIdx.x * 16 + j] = tb + x;
    if (mine + j < n) offsets[mine + j] = base + tb + x;
    x += v[j];
  }
  __syncthreads();
  const uint32_t lane = threadIdx.x & 31u;
  const uint64_t rows = (n - t0 < kScanTile) ? n - t0 : kScanTile;
  for (uint64_t r = threadIdx.x >> 5; r < rows; r += blockDim.x >> 5) {
    const uint32_t L = __ldg(len + t0 + r);
    const uint32_t* src = paths + (t0 + r) * pitch;
    uint32_t* dst = vertices + s_off[r];
    for (uint32_t t = lane; t < L; t += 32) dst[t] = src[t];
  }
}

}  // namespace

uint64_t paths_scan_tiles(uint64_t n) { return (n + kScanTile - 1) / kScanTile; }

cudaError_t launch_paths_scan(const uint32_t* lengths, uint64_t n, unsigned long long* tile_sum,
                              unsigned long long* total, cudaStream_t s) {
  const uint64_t nt = (n + kScanTile - 1) / kScanTile;
  if (nt) k_scan_tiles<<<(uint32_t)nt, 256, 0, s>>>(lengths, n, tile_sum);
  k_scan_tile_sums<<<1, 1024, 0, s>>>(tile_sum, nt, total);
  return cudaGetLastError();
}

cudaError_t launch_paths_pack(const uint32_t* lengths, uint64_t n, const unsigned long long* tile_off,
                              unsigned long long base, unsigned long long* offsets, const uint32_t* paths,
                              uint64_t pitch, uint32_t* vertices, cudaStream_t s) {
  const uint64_t nt = (n + kScanTile - 1) / kScanTile;
  if (nt) k_scan_apply<<<(uint32_t)nt, 256, 0, s>>>(lengths, n, tile_off, base, offsets, paths, pitch, vertices);
  return cudaGetLastError();
}

namespace {

__global__ void k_check_range(const uint32_t* a, uint64_t cnt, uint32_t n, uint32_t* bad) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < cnt; i += (uint64_t)gridDim.x * blockDim.x)
    if (a[i] >= n) { atomicOr(bad, 1u); return; }
}

__global__ void k_pool_reset(Params p) {
  const Pool& pl = p.pool;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  const uint64_t tid = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  for (uint64_t i = tid; i < pl.num_chunks; i += stride) pl.free_list[i] = (uint32_t)i;
  const uint64_t nring = (uint64_t)pl.nbuckets * pl.ring_len;
  for (uint64_t i = tid; i < nring; i += stride) pl.ring[i] = kEmpty;
  for (uint64_t i = tid; i < pl.nbuckets; i += stride) {
    pl.head[i * pl.hs] = 0;
    pl.cursor[i * pl.hs] = (i == 0 && p.direct.starts) ? p.direct.count : 0;  // direct start: W virtual positions
    pl.claim[i * pl.hs] = 0;
  }
  if (tid == 0) {
    *pl.free_top = (int)pl.num_chunks;
    p.ctr->steps = 0; p.ctr->visits = 0; p.ctr->truncated = 0; p.ctr->err = 0; p.ctr->done_ctas = 0;
    p.ctr->sent = 0;
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

int update_kernel_occupancy(uint32_t block, uint32_t ilp, uint32_t refill, uint32_t app, uint32_t P) {
  int nb = 0;
  const size_t dyn = (P + 1 <= kSmemBoundsCap) ? (size_t)(P + 1) * sizeof(uint32_t) : 0;
  (void)dyn;
  if (refill && app == 1) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_update_rf<1, 3, 1, 0, 0>, (int)block, 0);
  else if (refill) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_update_rf<0, 3, 1, 0, 0>, (int)block, 0);
  else if (ilp == 1) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_update<0, 3, 1, 1, 0>, (int)block, 0);
  else if (ilp == 4) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_update<0, 3, 4, 1, 0>, (int)block, 0);
  else cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_update<0, 3, 2, 1, 0>, (int)block, 0);
  return nb > 0 ? nb : 1;
}

// Augmented adjacency (LAY 1): adj[i] = {u, deg(u), row_ptr[u] lo, row_ptr[u] hi8 | slot(u) << 8} for u = col[i].
// .w = row_ptr[u] bits 32..39 | slot(u) << 8 (the visit-count slot of VIS 4, 0 without; offsets < 2^40).
__global__ void k_build_adj(const unsigned long long* __restrict__ row_ptr, const uint32_t* __restrict__ col,
                            uint64_t m, uint4* __restrict__ adj, const uint32_t* __restrict__ slot) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t u = col[i];
    const unsigned long long o = __ldg(row_ptr + u);
    const uint32_t dg = (uint32_t)(__ldg(row_ptr + u + 1) - o);
    const uint32_t sl = slot ? __ldg(slot + u) : 0u;
    adj[i] = make_uint4(u, dg, (uint32_t)o, (uint32_t)(o >> 32) | (sl << 8));
  }
}

cudaError_t launch_build_adj(const unsigned long long* row_ptr, const uint32_t* col, uint64_t m, uint4* adj,
                             const uint32_t* slot, cudaStream_t s) {
  if (!m) return cudaSuccess;
  k_build_adj<<<num_sms() * 8, 256, 0, s>>>(row_ptr, col, m, adj, slot);
  return cudaGetLastError();
}

// Compact augmented adjacency (LAY 2): words 3i..3i+2 = {u, row_ptr[u] lo32, row_ptr[u] hi8 | deg(u) << 8}
// for u = col[i] (the host checked row_ptr[n] < 2^40 and every degree < 2^24).
__global__ void k_build_adj12(const unsigned long long* __restrict__ row_ptr, const uint32_t* __restrict__ col,
                              uint64_t m, uint32_t* __restrict__ a12) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t u = col[i];
    const unsigned long long o = __ldg(row_ptr + u);
    const uint32_t dg = (uint32_t)(__ldg(row_ptr + u + 1) - o);
    a12[3 * i] = u;
    a12[3 * i + 1] = (uint32_t)o;
    a12[3 * i + 2] = (uint32_t)(o >> 32) | (dg << 8);
  }
}

cudaError_t launch_build_adj12(const unsigned long long* row_ptr, const uint32_t* col, uint64_t m, uint32_t* a12,
                               cudaStream_t s) {
  if (!m) return cudaSuccess;
  k_build_adj12<<<num_sms() * 8, 256, 0, s>>>(row_ptr, col, m, a12);
  return cudaGetLastError();
}

cudaError_t launch_insert_records(const Params& p, const uint4* recs, uint64_t count, cudaStream_t s) {
  if (!count) return cudaSuccess;
  uint64_t want = (count + 255) / 256;
  uint32_t grid = (uint32_t)std::min<uint64_t>(want, (uint64_t)num_sms() * 8);
  cudaFuncSetAttribute(k_insert_records, cudaFuncAttributeMaxDynamicSharedMemorySize, kSmemBoundsCap * 4);
  k_insert_records<<<grid, 256, bounds_smem(p), s>>>(p, recs, count, nullptr);
  return cudaGetLastError();
}

cudaError_t launch_insert_records_dev(const Params& p, const uint4* recs, const unsigned long long* dcount,
                                      cudaStream_t s) {
  cudaFuncSetAttribute(k_insert_records, cudaFuncAttributeMaxDynamicSharedMemorySize, kSmemBoundsCap * 4);
  k_insert_records<<<num_sms() * 8, 256, bounds_smem(p), s>>>(p, recs, 0, dcount);
  return cudaGetLastError();
}

cudaError_t launch_pack(const Params& p, uint32_t bucket, uint4* out, uint64_t count, cudaStream_t s) {
  if (!count) return cudaSuccess;
  uint64_t want = (count + 255) / 256;
  uint32_t grid = (uint32_t)std::min<uint64_t>(want, (uint64_t)num_sms() * 8);
  k_pack<<<grid, 256, 0, s>>>(p, bucket, out);
  return cudaGetLastError();
}

cudaError_t launch_init(const Params& p, const uint32_t* starts, uint64_t W, uint64_t first_row, cudaStream_t s) {
  uint64_t want = (W + 255) / 256;
  uint32_t grid = (uint32_t)std::min<uint64_t>(want ? want : 1, (uint64_t)num_sms() * 8);
  cudaFuncSetAttribute(k_init, cudaFuncAttributeMaxDynamicSharedMemorySize, kSmemBoundsCap * 4);
  k_init<<<grid, 256, bounds_smem(p), s>>>(p, starts, W, first_row);
  return cudaGetLastError();
}

template <int APP, int GM, int ILP, int LAY, int VIS>
void launch_update_t(const Params& p, uint32_t k, uint32_t grid, uint32_t block, cudaStream_t s) {
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(k_update<APP, GM, ILP, LAY, VIS>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         kSmemBoundsCap * 4);
    attr = true;
  }
  k_update<APP, GM, ILP, LAY, VIS><<<grid, block, bounds_smem(p), s>>>(p, k);
}

template <int APP, int GM, int LAY, int VIS, int CONT>
void launch_update_rf_t(const Params& p, uint32_t k, uint32_t grid, uint32_t block, cudaStream_t s) {
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(k_update_rf<APP, GM, LAY, VIS, CONT>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         kSmemBoundsCap * 4);
    attr = true;
  }
  k_update_rf<APP, GM, LAY, VIS, CONT><<<grid, block, bounds_smem(p), s>>>(p, k);
}

template <int APP, int GM, int LAY, int VIS>
void launch_update_rf(const Params& p, uint32_t k, uint32_t grid, uint32_t block, cudaStream_t s) {
  if constexpr (LAY == 0) {
    if (p.cont.table) {
      launch_update_rf_t<APP, GM, LAY, VIS, 1>(p, k, grid, block, s);
      return;
    }
  }
  launch_update_rf_t<APP, GM, LAY, VIS, 0>(p, k, grid, block, s);
}

template <int APP, int GM, int LAY, int VIS>
void launch_update_ilp(const Params& p, uint32_t k, uint32_t grid, uint32_t block, cudaStream_t s) {
  if (p.refill) {
    launch_update_rf<APP, GM, LAY, VIS>(p, k, grid, block, s);
    return;
  }
  switch (p.ilp) {
    case 1: launch_update_t<APP, GM, 1, LAY, VIS>(p, k, grid, block, s); break;
    case 4: launch_update_t<APP, GM, 4, LAY, VIS>(p, k, grid, block, s); break;
    default: launch_update_t<APP, GM, 2, LAY, VIS>(p, k, grid, block, s); break;
  }
}

template <int APP, int VIS>
void launch_update_app(const Params& p, uint32_t k, uint32_t grid, uint32_t block, cudaStream_t s) {
  const bool adj = p.wk.adj != nullptr, adj12 = p.wk.adj12 != nullptr;
  if (p.gather_mode == 0) {
    if (adj) launch_update_ilp<APP, 0, 1, VIS>(p, k, grid, block, s);
    else if (adj12) launch_update_ilp<APP, 0, 2, VIS>(p, k, grid, block, s);
    else launch_update_ilp<APP, 0, 0, VIS>(p, k, grid, block, s);
  } else {
    if (adj) launch_update_ilp<APP, 3, 1, VIS>(p, k, grid, block, s);
    else if (adj12) launch_update_ilp<APP, 3, 2, VIS>(p, k, grid, block, s);
    else launch_update_ilp<APP, 3, 0, VIS>(p, k, grid, block, s);
  }
}

template <int VIS>
void launch_update_vis(const Params& p, uint32_t k, uint32_t grid, uint32_t block, cudaStream_t s) {
  if (p.wk.app == 0) launch_update_app<0, VIS>(p, k, grid, block, s);
  else if (p.wk.app == 1) launch_update_app<1, VIS>(p, k, grid, block, s);
  else launch_update_app<2, VIS>(p, k, grid, block, s);
}

template <int APP>
void launch_update_vis3(const Params& p, uint32_t k, uint32_t grid, uint32_t block, cudaStream_t s) {
  if (p.wk.adj) launch_update_ilp<APP, 3, 1, 3>(p, k, grid, block, s);
  else launch_update_ilp<APP, 3, 2, 3>(p, k, grid, block, s);
}

cudaError_t launch_update(const Params& p, uint32_t k, uint32_t grid, uint32_t block, cudaStream_t s) {
  if (p.wk.vhot) {  // the host selects VIS 4 only with the ADJ layout built with slots and gather_mode 3
    if (p.wk.app == 0) launch_update_ilp<0, 3, 1, 4>(p, k, grid, block, s);
    else if (p.wk.app == 1) launch_update_ilp<1, 3, 1, 4>(p, k, grid, block, s);
    else launch_update_ilp<2, 3, 1, 4>(p, k, grid, block, s);
  } else if (p.wk.visits16) {  // the host selects VIS 3 only with an augmented layout and gather_mode 3
    if (p.wk.app == 0) launch_update_vis3<0>(p, k, grid, block, s);
    else if (p.wk.app == 1) launch_update_vis3<1>(p, k, grid, block, s);
    else launch_update_vis3<2>(p, k, grid, block, s);
  } else if (p.wk.visits32) launch_update_vis<2>(p, k, grid, block, s);
  else if (p.wk.visits) launch_update_vis<1>(p, k, grid, block, s);
  else launch_update_vis<0>(p, k, grid, block, s);
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

cudaError_t launch_snapshot(const unsigned long long* hc, uint64_t nb, uint32_t hs, const Counters* ctr,
                            const int* free_top, unsigned long long* out_hc, Counters* out_ctr, int* out_free,
                            cudaStream_t s) {
  k_snapshot<<<1, 256, 0, s>>>(hc, nb, hs, ctr, free_top, out_hc, out_ctr, out_free);
  return cudaGetLastError();
}

cudaError_t launch_compact_rows(const uint32_t* paths, const uint32_t* lengths, uint64_t pitch, uint64_t stride,
                                uint64_t n, uint32_t* out, cudaStream_t s) {
  if (!n) return cudaSuccess;
  k_compact_rows<<<num_sms() * 8, 256, 0, s>>>(paths, lengths, pitch, stride, n, out);
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

struct TableSet {
  uint32_t idx[kTableSetMax], val[kTableSetMax];
};
__global__ void k_table_set(uint32_t* table, TableSet ts, uint32_t count) {
  if (threadIdx.x < count) table[ts.idx[threadIdx.x]] = ts.val[threadIdx.x];
}

__global__ void k_widen(const uint32_t* __restrict__ src, unsigned long long* __restrict__ dst, uint64_t n) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    dst[i] = src[i];
}

cudaError_t launch_table_set(uint32_t* table, const uint32_t* idx, const uint32_t* val, uint32_t count,
                             cudaStream_t s) {
  if (!count) return cudaSuccess;
  if (count > kTableSetMax) return cudaErrorInvalidValue;
  TableSet ts;
  for (uint32_t i = 0; i < count; ++i) {
    ts.idx[i] = idx[i];
    ts.val[i] = val[i];
  }
  k_table_set<<<1, 32, 0, s>>>(table, ts, count);
  return cudaGetLastError();
}

// VIS 3: counts[v] = hub(v) ? visits32[v] : half v & 1 of visits16[v >> 1]; the sum of all counts goes to
// *sum (compared on the host with the number of path entries: any 16-bit wrap makes it fall short).
__global__ void k_widen16(const uint32_t* __restrict__ v16, const uint32_t* __restrict__ v32,
                          const unsigned long long* __restrict__ row_ptr, uint32_t hub_deg,
                          unsigned long long* __restrict__ dst, uint64_t n, unsigned long long* sum) {
  unsigned long long acc = 0;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t dg = (uint32_t)(row_ptr[i + 1] - row_ptr[i]);
    const uint32_t c = dg >= hub_deg ? v32[i] : ((v16[i >> 1] >> ((i & 1) * 16)) & 0xFFFFu);
    dst[i] = c;
    acc += c;
  }
  using BR = cub::BlockReduce<unsigned long long, 256>;
  __shared__ typename BR::TempStorage tmp;
  acc = BR(tmp).Sum(acc);
  if (threadIdx.x == 0 && acc) atomicAdd(sum, acc);
}

// Exact recount from the path matrix (the fallback after a detected 16-bit wrap): counts[paths[w][t]] += 1
// for t < lengths[w], a warp per row.
__global__ void k_recount(const uint32_t* __restrict__ paths, uint64_t pitch, const uint32_t* __restrict__ lengths,
                          uint64_t W, unsigned long long* __restrict__ dst) {
  const uint64_t lane = threadIdx.x & 31u;
  for (uint64_t w = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; w < W;
       w += ((uint64_t)gridDim.x * blockDim.x) >> 5) {
    const uint32_t L = lengths[w];
    for (uint64_t t = lane; t < L; t += 32) atomicAdd(dst + paths[w * pitch + t], 1ull);
  }
}

cudaError_t launch_widen16(const uint32_t* v16, const uint32_t* v32, const unsigned long long* row_ptr,
                           uint32_t hub_deg, unsigned long long* dst, uint64_t n, unsigned long long* sum,
                           cudaStream_t s) {
  if (!n) return cudaSuccess;
  k_widen16<<<num_sms() * 8, 256, 0, s>>>(v16, v32, row_ptr, hub_deg, dst, n, sum);
  return cudaGetLastError();
}

cudaError_t launch_recount(const uint32_t* paths, uint64_t pitch, const uint32_t* lengths, uint64_t W,
                           unsigned long long* dst, cudaStream_t s) {
  if (!W) return cudaSuccess;
  k_recount<<<num_sms() * 8, 256, 0, s>>>(paths, pitch, lengths, W, dst);
  return cudaGetLastError();
}

// Compressed partition transfer (lt_config.ooc_compress): a warp per block of 32 column entries. Lane i
// extracts its w-bit zigzag delta (bits [i w, (i+1) w) of the block's payload; lane 0's delta is 0), the
// warp's inclusive prefix sum (mod 2^32) plus the block's first value gives entry i.
__global__ void k_decode_cols(const uint2* __restrict__ hdr, const uint32_t* __restrict__ pay, uint64_t len,
                              uint32_t* __restrict__ out) {
  const uint32_t lane = threadIdx.x & 31u;
  const uint64_t nblk = (len + 31) >> 5;
  for (uint64_t j = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; j < nblk;
       j += ((uint64_t)gridDim.x * blockDim.x) >> 5) {
    const uint2 h = hdr[j];
    const uint32_t w = hdr[j + 1].y - h.y;
    uint32_t z = 0;
    if (w) {
      const uint32_t bit = lane * w, wi = bit >> 5, sh = bit & 31u;
      uint64_t x = pay[h.y + wi];
      if (sh + w > 32) x |= (uint64_t)pay[h.y + wi + 1] << 32;
      z = (uint32_t)(x >> sh) & (w == 32 ? 0xFFFFFFFFu : ((1u << w) - 1u));
    }
    uint32_t v = (z >> 1) ^ (0u - (z & 1u));  // unzigzag: the delta mod 2^32
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(kFull, v, o);
      if (lane >= (uint32_t)o) v += y;
    }
    const uint64_t i = (j << 5) + lane;
    if (i < len) out[i] = h.x + v;
  }
}

cudaError_t launch_decode_cols(const uint2* hdr, const uint32_t* pay, uint64_t len, uint32_t* out, cudaStream_t s) {
  if (!len) return cudaSuccess;
  const uint64_t warps = (len + 31) >> 5;
  const uint32_t grid = (uint32_t)std::min<uint64_t>((warps + 7) / 8, (uint64_t)num_sms() * 16);
  k_decode_cols<<<grid, 256, 0, s>>>(hdr, pay, len, out);
  return cudaGetLastError();
}

// VIS 4 per-vertex table: vinfo[v] = {row_ptr[v] lo32, row_ptr[v] hi8 | slot[v] << 8, deg(v), 0}
__global__ void k_build_vinfo(const unsigned long long* __restrict__ row_ptr, const uint32_t* __restrict__ slot,
                              uint64_t n, uint4* __restrict__ vinfo) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    const unsigned long long o = row_ptr[i];
    vinfo[i] = make_uint4((uint32_t)o, (uint32_t)(o >> 32) | (slot[i] << 8), (uint32_t)(row_ptr[i + 1] - o), 0u);
  }
}

cudaError_t launch_build_vinfo(const unsigned long long* row_ptr, const uint32_t* slot, uint64_t n, uint4* vinfo,
                               cudaStream_t s) {
  if (!n) return cudaSuccess;
  k_build_vinfo<<<num_sms() * 8, 256, 0, s>>>(row_ptr, slot, n, vinfo);
  return cudaGetLastError();
}

// VIS 4: counts[v] = visits32[v] + (slot[v] ? vhot[slot[v]] : 0)
__global__ void k_widen_slots(const uint32_t* __restrict__ cold, const uint32_t* __restrict__ hot,
                              const uint32_t* __restrict__ slot, unsigned long long* __restrict__ dst, uint64_t n) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t sl = slot[i];
    dst[i] = (unsigned long long)cold[i] + (sl ? hot[hot_index(sl)] : 0u);
  }
}

cudaError_t launch_widen_slots(const uint32_t* cold, const uint32_t* hot, const uint32_t* slot, unsigned long long* dst,
                               uint64_t n, cudaStream_t s) {
  if (!n) return cudaSuccess;
  k_widen_slots<<<num_sms() * 8, 256, 0, s>>>(cold, hot, slot, dst, n);
  return cudaGetLastError();
}

cudaError_t launch_widen(const uint32_t* src, unsigned long long* dst, uint64_t n, cudaStream_t s) {
  if (!n) return cudaSuccess;
  k_widen<<<num_sms() * 8, 256, 0, s>>>(src, dst, n);
  return cudaGetLastError();
}

cudaError_t launch_spill(const Params& p, const SpillList& list, uint32_t count, uint4* store, cudaStream_t s) {
  if (!count) return cudaSuccess;
  k_spill<<<count, 256, 0, s>>>(p, list, store);
  return cudaGetLastError();
}

cudaError_t launch_reload(const Params& p, const SpillList& list, uint32_t count, const uint4* store, cudaStream_t s) {
  if (!count) return cudaSuccess;
  k_reload<<<count, 256, 0, s>>>(p, list, store);
  return cudaGetLastError();
}

// Diagnostic (tests/test_gpu_philox.py, SURVEY.md §4 pin P2): the update kernels' own Philox4x32-10 on
// given counters and keys, so the device RNG can be compared with cuRAND's curand_Philox4x32_10.
__global__ void k_philox_blocks(const uint4* __restrict__ ctr, const uint2* __restrict__ key, uint4* __restrict__ out,
                                uint64_t n) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    out[i] = philox10(ctr[i], key[i].x, key[i].y);
}

cudaError_t launch_philox_blocks(const uint4* ctr, const uint2* key, uint4* out, uint64_t n, cudaStream_t s) {
  if (!n) return cudaSuccess;
  k_philox_blocks<<<num_sms() * 4, 256, 0, s>>>(ctr, key, out, n);
  return cudaGetLastError();
}

cudaError_t launch_pool_reset(const Params& p, cudaStream_t s) {
  k_pool_reset<<<num_sms() * 4, 256, 0, s>>>(p);
  return cudaGetLastError();
}

}  // namespace lt
