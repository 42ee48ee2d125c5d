// lt_internal.h — device-side state shared by the host scheduler (lt_abi.cpp) and the kernels
// (lt_kernels.cu). Not part of the ABI.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace lt {

constexpr uint32_t kEmpty = 0xFFFFFFFFu;   // empty ring slot / unused path slot
constexpr uint32_t kErrOOM = 1u;           // device error bits
constexpr uint32_t kErrRing = 2u;
constexpr uint32_t kErrPeer = 4u;          // a peer receive buffer overflowed
constexpr uint32_t kSpilled = 0xFFFFFFFEu; // ring slot of a chunk evicted to host memory (walk spill)

// A walk record (D5): 16 bytes, one 128-bit load/store.
//   x = local walk index (row of the path matrix; walk_id = first_walk_id + x)
//   y = current_vertex, z = walked_steps, w = reserved (0)

// Walk pool (a6): `slots` is an arena of num_chunks chunks of C records.
// Bucket k is the position range [head[k], cursor[k]) (monotone u64 counters); position pos lives
// in chunk ring[k*ring_len + (pos/C) % ring_len] at offset pos % C. Ring slots are installed on
// demand: exactly once per chunk, by the writer whose claim holds the chunk's first slot.
struct Pool {
  uint4* slots;
  uint32_t C, c_shift;
  uint32_t num_chunks;            // + 1 trash chunk at index num_chunks (writes after OOM)
  uint32_t* ring;
  uint32_t ring_len;
  uint32_t nbuckets;              // P partition buckets + one send bucket per other rank
  // Bucket b's head / cursor / claim are head[b * hs], cursor[b * hs], claim[b * hs] (one block of hs
  // u64 per bucket: cursor = head + 1, claim = head + 2). hs = 32 (256 B) while the buckets are few, so
  // every bucket's cursor — the target of every insertion atomic — has its own L2 line and slice.
  unsigned long long* head;
  unsigned long long* cursor;
  unsigned long long* claim;      // refill claims within a launch (== head between launches)
  uint32_t hs;
  uint32_t* free_list;            // [num_chunks]
  int* free_top;
};

struct Walk {
  // The graph the update launch gathers from. Resident mode: the whole CSR (vbase = ebase = 0).
  // Out-of-core mode: one partition's slice in a graph-pool block, row_ptr[0] is vertex vbase's
  // offset and col[0] is CSR entry ebase (or the whole CSR mapped from pinned host for zero copy).
  const unsigned long long* row_ptr;
  const uint32_t* col;
  uint32_t vbase;
  unsigned long long ebase;
  const uint4* adj;               // [m] augmented adjacency {u, deg(u), row_ptr[u]} or nullptr
  const uint32_t* adj12;          // [3m] compact augmented adjacency (12 B per entry) or nullptr
  const uint32_t* bounds;         // [P+1]
  uint32_t P;
  uint32_t* paths;
  uint64_t stride;                // logical row length: l+1 (DeepWalk) or L_max+1 (PPR)
  uint64_t pitch;                 // physical row pitch in u32: stride rounded up to 8 (32-B sectors)
  uint32_t path_mode;             // 0 buffered full-sector stores, 1 one store per step, 2 no stores (ablation)
  uint32_t* lengths;
  uint64_t first_walk_id;
  uint32_t seed_lo, seed_hi;
  uint32_t app, length, T, lmax;  // app: 0 DeepWalk, 1 PPR, 2 PageRank (random walk with restart)
  uint32_t n;                     // |V|: a PageRank restart draws its vertex from [0, n)
  unsigned long long* visits;     // [n] per-vertex visit counts or nullptr (off)
  uint32_t* visits32;             // [n] narrow counters used instead while every count fits in u32
                                  // (W * stride < 2^32); widened into `visits` at the end of lt_run;
                                  // with visits16: the hub counters (degree >= hub_deg)
  uint32_t* visits16;             // [ceil(n/2)] paired 16-bit counters of the non-hub vertices, or nullptr
  uint32_t hub_deg;               // degree from which a vertex counts in visits32 (visits16 on)
  uint32_t* vhot;                 // VIS 4: [2^24] counters by degree slot (the ADJ entry's .w >> 8), or nullptr
  const uint4* vinfo;             // VIS 4: [n] {off lo32, off hi8 | slot << 8, deg, 0} per vertex
};

constexpr uint32_t kHotSlots = 1u << 24;  // VIS 4: slots 1 .. kHotSlots - 1 (24 bits of the ADJ entry's .w)
// VIS 4 counter index of slot s: the kHotSpread hottest slots one per 128-B line (their REDs would
// otherwise serialise on a few L2 lines), the rest packed densely after them
constexpr uint32_t kHotSpread = 1u << 15;
__host__ __device__ inline uint64_t hot_index(uint32_t s) {
  return s < kHotSpread ? (uint64_t)s * 32 : (uint64_t)kHotSpread * 32 + (s - kHotSpread);
}
constexpr uint64_t kHotWords = (uint64_t)kHotSpread * 32 + kHotSlots;

struct Counters {
  unsigned long long steps, visits, truncated;
  uint32_t err;
  uint32_t done_ctas;
  unsigned long long sent;  // records appended to other ranks' receive buffers (peer exchange)
};

// Range ownership across ranks (north star 8-GPU mode): this rank owns partitions
// [own_lo, own_hi); a walk whose next partition q is owned elsewhere goes to the send bucket
// P + owner[q]. world == 1: own_lo = 0, own_hi = P, no send buckets.
struct Owner {
  uint32_t own_lo, own_hi;
  const uint16_t* owner;  // [P] rank of each partition (nullptr when world == 1)
};

// Resident-neighbour continuation (out-of-core mode): table[q] = graph-pool block
// holding partition q, ready and safe to read for the whole launch, or kEmpty. A walk that leaves the
// launched partition for a partition in the table keeps stepping through that block's view instead of
// being appended to a bucket. table == nullptr: off.
struct Cont {
  const uint32_t* table;          // [P]
  const char* gpool;              // block b at gpool + b * block_bytes: row_ptr slice, col slice at rp_bytes
  uint64_t block_bytes, rp_bytes;
};

// Direct start (one partition, one rank, every walk admitted at once): bucket 0 holds the W new walks
// as VIRTUAL positions [0, W) — no record is written by k_init; the lane-refill kernel builds the
// record of position j in registers as {j, starts[j], 0, 0}. Positions past W (none with one
// partition: a walk never leaves it) would be real slots. starts == nullptr: off.
struct Direct {
  const uint32_t* starts;
  unsigned long long count;
};

// Peer exchange (lt_exchange_attach; the multi-GPU mode without pack + all-to-all): a walk whose
// next partition is owned by rank q is appended by the insertion epilogue straight into rank q's
// receive buffer over peer memory (NVLink), with one atomic per (warp, destination rank) on q's
// cursor. Receive buffers and cursors are double-buffered by superstep parity `epoch`, so senders of
// superstep s+1 never touch the buffer a receiver is still draining from superstep s.
// recv == nullptr: off (walks for other ranks go to the local send buckets).
struct Peer {
  uint4* const* recv;                    // [2 * world]: buffer of rank q for epoch e at [e * world + q]
  unsigned long long* const* cursor;     // [2 * world]: same indexing, one u64 each
  unsigned long long cap;                // records per buffer
  uint32_t epoch;
};

struct Params {
  Walk wk;
  Peer peer;
  Cont cont;
  Pool pool;
  Counters* ctr;
  Owner own;
  Direct direct;
  uint32_t insert_mode;
  uint32_t gather_mode;
  uint32_t ilp;
  uint32_t refill;  // 0: batch kernel (k_update), 1: lane refill (k_update_rf)
  unsigned long long tail_cap;  // an update launch consumes [head, min(cursor, tail_cap)) (walk spill); ~0 otherwise
  uint32_t sys_fence;           // kernels end with a system-scope fence: they wrote peer memory (paths on the home rank)
};

// Walk spill (lt_config.walk_spill): chunks moved between the device pool and host memory per launch.
constexpr uint32_t kSpillBatch = 64;
struct SpillList {
  uint32_t bucket[kSpillBatch];
  uint32_t slot[kSpillBatch];             // host store slot
  unsigned long long chunk[kSpillBatch];  // chunk index within the bucket (position / C)
};

// launchers (lt_kernels.cu); all asynchronous on `s`
// walks [first_row, first_row + W) from starts[0..W): records, visit counts, insertion (a2)
cudaError_t launch_init(const Params& p, const uint32_t* starts, uint64_t W, uint64_t first_row, cudaStream_t s);
cudaError_t launch_insert_records(const Params& p, const uint4* recs, uint64_t count, cudaStream_t s);
// the same with the record count read from device memory (fused superstep of the peer exchange)
cudaError_t launch_insert_records_dev(const Params& p, const uint4* recs, const unsigned long long* dcount,
                                      cudaStream_t s);
cudaError_t launch_pack(const Params& p, uint32_t bucket, uint4* out, uint64_t count, cudaStream_t s);
cudaError_t launch_update(const Params& p, uint32_t k, uint32_t grid, uint32_t block, cudaStream_t s);
cudaError_t launch_finalize_paths(const Params& p, uint64_t W, cudaStream_t s);
cudaError_t launch_gather_rows(const Params& p, const unsigned long long* rows, uint64_t count,
                               uint32_t* out_paths, uint32_t* out_lengths, cudaStream_t s);
cudaError_t launch_snapshot(const unsigned long long* hc, uint64_t nb, uint32_t hs, const Counters* ctr, const int* free_top,
                            unsigned long long* out_hc, Counters* out_ctr, int* out_free, cudaStream_t s);
cudaError_t launch_compact_rows(const uint32_t* paths, const uint32_t* lengths, uint64_t pitch, uint64_t stride,
                                uint64_t n, uint32_t* out, cudaStream_t s);
cudaError_t launch_check_col(const uint32_t* col, uint64_t m, uint32_t n, uint32_t* bad, cudaStream_t s);
cudaError_t launch_check_starts(const uint32_t* starts, uint64_t W, uint32_t n, uint32_t* bad, cudaStream_t s);
cudaError_t launch_pool_reset(const Params& p, cudaStream_t s);
cudaError_t launch_philox_blocks(const uint4* ctr, const uint2* key, uint4* out, uint64_t n, cudaStream_t s);
// walk spill: chunks list[0..count) -> their host slots of `store` (the mapped host store; ring slots marked
// kSpilled, device chunks freed) / host slots -> fresh device chunks installed in the ring
cudaError_t launch_spill(const Params& p, const SpillList& list, uint32_t count, uint4* store, cudaStream_t s);
cudaError_t launch_reload(const Params& p, const SpillList& list, uint32_t count, const uint4* store, cudaStream_t s);
// compact path output: (1) tile sums + their exclusive scan (total -> *total); (2) offsets[i] = base +
// exclusive prefix of lengths for i < n, rows packed into vertices (indexed from 0 for this range)
uint64_t paths_scan_tiles(uint64_t n);  // tile_sum entries launch_paths_scan needs
cudaError_t launch_paths_scan(const uint32_t* lengths, uint64_t n, unsigned long long* tile_sum,
                              unsigned long long* total, cudaStream_t s);
cudaError_t launch_paths_pack(const uint32_t* lengths, uint64_t n, const unsigned long long* tile_off,
                              unsigned long long base, unsigned long long* offsets, const uint32_t* paths,
                              uint64_t pitch, uint32_t* vertices, cudaStream_t s);
cudaError_t launch_table_set(uint32_t* table, const uint32_t* idx, const uint32_t* val, uint32_t count,
                             cudaStream_t s);  // table[idx[i]] = val[i], count <= kTableSetMax
constexpr uint32_t kTableSetMax = 32;
cudaError_t launch_widen(const uint32_t* src, unsigned long long* dst, uint64_t n, cudaStream_t s);
cudaError_t launch_build_vinfo(const unsigned long long* row_ptr, const uint32_t* slot, uint64_t n, uint4* vinfo,
                               cudaStream_t s);
cudaError_t launch_widen_slots(const uint32_t* cold, const uint32_t* hot, const uint32_t* slot, unsigned long long* dst,
                               uint64_t n, cudaStream_t s);
cudaError_t launch_decode_cols(const uint2* hdr, const uint32_t* pay, uint64_t len, uint32_t* out, cudaStream_t s);
cudaError_t launch_widen16(const uint32_t* v16, const uint32_t* v32, const unsigned long long* row_ptr,
                           uint32_t hub_deg, unsigned long long* dst, uint64_t n, unsigned long long* sum,
                           cudaStream_t s);
cudaError_t launch_recount(const uint32_t* paths, uint64_t pitch, const uint32_t* lengths, uint64_t W,
                           unsigned long long* dst, cudaStream_t s);
cudaError_t launch_build_adj(const unsigned long long* row_ptr, const uint32_t* col, uint64_t m, uint4* adj,
                             const uint32_t* slot, cudaStream_t s);
cudaError_t launch_build_adj12(const unsigned long long* row_ptr, const uint32_t* col, uint64_t m, uint32_t* a12,
                               cudaStream_t s);
// resident blocks per SM of the update kernel the launch uses (refill: 0 batch, 1 lane refill)
int update_kernel_occupancy(uint32_t block, uint32_t ilp, uint32_t refill, uint32_t app, uint32_t P);
uint32_t update_smem_bounds_cap();             // max P whose bounds are staged in shared memory

}  // namespace lt
