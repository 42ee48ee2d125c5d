// lt_ctx.h — the library context behind the opaque lt_ctx handle (private to csrc/).
#pragma once
#include "lt.h"
#include "lt_internal.h"

#include <algorithm>
#include <map>
#include <string>
#include <vector>

struct lt_ctx;

namespace lt {

lt_status fail(lt_status s, const std::string& msg);

// Device memory of the library's pools ("the library sub-allocates all pools from it
// once"): from the caller-owned arena (lt_config.arena) when one is given — a bump allocator, 256-B
// aligned; freeing inside the arena is a no-op and lt_graph_load* resets it — else cudaMalloc.
cudaError_t dmalloc(lt_ctx* ctx, void** p, size_t bytes);
void dfree(lt_ctx* ctx, void* p);
void arena_track(lt_ctx* ctx, void** p, size_t* cap);  // ensure() buffers: nulled when the arena resets

template <class T>
cudaError_t ensure(lt_ctx* ctx, T*& p, size_t& cap, size_t count) {
  if (count <= cap && p) return cudaSuccess;
  if (p) dfree(ctx, p);
  p = nullptr;
  cap = 0;
  cudaError_t e = dmalloc(ctx, (void**)&p, std::max<size_t>(count, 1) * sizeof(T));
  if (e == cudaSuccess) {
    cap = count;
    arena_track(ctx, (void**)&p, &cap);
  }
  return e;
}

// Out-of-core graph state: the CSR lives in
// pinned, mapped host memory (G_cpu); a graph pool of m_g equal blocks caches partitions on the
// device; a load stream copies partitions in while the compute stream runs resident ones.
struct OutOfCore {
  bool on = false;
  unsigned long long* h_row_ptr = nullptr;  // pinned + mapped, n+1
  uint32_t* h_col = nullptr;                // pinned + mapped, m
  unsigned long long* d_map_row_ptr = nullptr;  // device views of the mapped host arrays (zero copy)
  uint32_t* d_map_col = nullptr;
  char* d_gpool = nullptr;   // m_g blocks of block_bytes
  size_t block_bytes = 0;
  size_t rp_bytes = 0;       // bytes reserved for the row_ptr slice at the start of each block
  uint32_t m_g = 0;
  std::vector<int> block_of;   // partition -> block (-1: not resident)
  std::vector<int> part_in;    // block -> partition (-1: free)
  std::vector<uint64_t> loaded_at;  // block -> load sequence number (FIFO eviction)
  std::vector<cudaEvent_t> ev_ready, ev_used;  // per block: load finished / last compute use
  cudaStream_t load_stream = nullptr;
  // resident-neighbour continuation (f4): device table partition -> block (kEmpty if not usable) and
  // its host mirror
  uint32_t* d_table = nullptr;
  std::vector<uint32_t> table;
  // compressed column slices (lt_config.ooc_compress): partition k's slice in blocks of 32 entries, header
  // j = {first value, payload word offset from the partition's first payload word} (nblk + 1 headers, the
  // last a sentinel), payload = the block's zigzag deltas bit-packed at width w = next offset - offset
  bool comp = false;
  uint2* h_chdr = nullptr;                 // pinned: every partition's headers
  uint32_t* h_cpay = nullptr;              // pinned: every partition's payload words
  std::vector<uint64_t> chdr_at, cpay_at;  // per partition: first header / first payload word
  std::vector<uint8_t> craw;               // per partition: 1 = copied raw (compression saves nothing)
  char* d_cstage = nullptr;                // device staging of one partition's compressed slice
  size_t cstage_bytes = 0;
  uint64_t comp_bytes = 0;
};

// Walk spill (lt_config.walk_spill): the walk pool keeps at most its
// num_chunks chunks on the device; full chunks of buckets with the fewest pending walks are evicted to a
// pinned, MAPPED host store (PAPER.md:118 "evict a batch when full", :202 "the same way") and loaded back
// before their partition is computed. The copies are kernels (k_spill / k_reload, a block per chunk)
// that read and write the host store through its device mapping: no staging buffers and no per-chunk
// cudaMemcpy calls (a 128-KB memcpy ran at ~40 % of the link, measured).
struct Spill {
  bool on = false;
  uint4* h_store = nullptr;                 // pinned + mapped host chunk slots (host_cap x C records)
  uint4* d_store = nullptr;                 // its device view
  uint64_t host_cap = 0;
  std::vector<uint32_t> host_free;          // free host slots
  std::vector<std::map<uint64_t, uint32_t>> spilled;  // per bucket: chunk index -> host slot
  uint64_t host_used = 0;
  int64_t free_chunks = 0;                  // host mirror of the device free stack, kept exact between snapshots
};

// Per-phase timing ("update vs reshuffle vs loading"): CUDA-event pairs
// around the transfers of a phase on its own stream, summed at the end of lt_run (with lt_config.timing).
struct PhaseEvents {
  std::vector<cudaEvent_t> ev;
  size_t n = 0;  // events in use (pairs)
  cudaError_t begin(cudaStream_t s) {
    while (ev.size() < n + 2) {
      cudaEvent_t e;
      cudaError_t r = cudaEventCreate(&e);
      if (r != cudaSuccess) return r;
      ev.push_back(e);
    }
    return cudaEventRecord(ev[n], s);
  }
  cudaError_t end(cudaStream_t s) {
    cudaError_t r = cudaEventRecord(ev[n + 1], s);
    n += 2;
    return r;
  }
  cudaError_t total_ms(double* out) {  // sums and resets
    double t = 0;
    for (size_t i = 0; i + 1 < n; i += 2) {
      float ms = 0;
      cudaError_t r = cudaEventElapsedTime(&ms, ev[i], ev[i + 1]);
      if (r != cudaSuccess) return r;
      t += ms;
    }
    n = 0;
    *out = t;
    return cudaSuccess;
  }
  void destroy() {
    for (auto e : ev) cudaEventDestroy(e);
    ev.clear();
    n = 0;
  }
};

// NVTX ranges around the scheduler's phases (header-only NVTX3; a profiler shows them, free otherwise)
struct Range {
  explicit Range(const char* name);
  ~Range();
};

}  // namespace lt

struct lt_ctx {
  lt_config cfg{};
  cudaStream_t stream = nullptr;
  int num_sms = 148;
  int occ = 1;
  uint32_t block = 256;
  // graph
  bool graph_loaded = false;
  uint32_t n = 0;
  uint64_t m = 0;
  uint32_t P = 0;
  uint32_t nb = 0;             // buckets: P + (world > 1 ? world : 0)
  uint32_t rank = 0, world = 1, own_lo = 0, own_hi = 0;
  uint16_t* d_owner = nullptr;  // [P] owner rank per partition (world > 1)
  unsigned long long* d_row_ptr = nullptr;  // [n+1], the whole row_ptr (global offsets)
  uint32_t* d_col = nullptr;                // CSR entries [e_lo, e_hi): d_col[0] is entry e_lo
  uint64_t e_lo = 0, e_hi = 0;              // edges of the vertices this rank owns ([0, m) when world == 1)
  bool own_graph = false;
  uint4* d_adj = nullptr;  // augmented adjacency (layout ADJ), owned
  size_t adj_cap = 0;
  uint32_t* d_adj12 = nullptr;  // compact augmented adjacency (layout ADJ12, 3 words per entry), owned
  size_t adj12_cap = 0;
  std::vector<uint32_t> h_bounds;
  uint32_t* d_bounds = nullptr;
  size_t bounds_cap = 0;
  lt::OutOfCore ooc;
  lt::Spill spill;
  lt::PhaseEvents load_ev, xfer_ev;  // graph loads (load stream), walk-spill copy kernels (compute stream)
  // caller-owned arena (lt_config.arena): [arena, arena + arena_size), bump pointer arena_top; buffers
  // from ensure() registered in arena_bufs are dropped when a graph load resets the arena to arena_mark
  char* arena = nullptr;
  size_t arena_size = 0, arena_top = 0, arena_mark = 0, arena_peak = 0;
  std::vector<std::pair<void**, size_t*>> arena_bufs;
  // paths on the home rank (lt_paths_attach): this rank's path entries and lengths go straight into the
  // home rank's matrix over peer memory
  uint32_t* home_paths = nullptr;
  uint32_t* home_lengths = nullptr;
  uint64_t home_cap = 0;  // u32 entries of home_paths
  bool is_home = false;   // other ranks write into this rank's matrix (lt_paths_buffers was called)
  // walks
  bool walks_ready = false;
  bool ran = false;
  bool padded = false;  // path slots past each length hold 0xFFFFFFFF (done lazily, before a copy-out)
  bool snap_valid = false;  // h_hc / h_ctr / h_free mirror the device (no pool-changing launch since)
  uint64_t W = 0, first = 0, seed = 0;
  lt_app app = LT_APP_DEEPWALK;
  uint32_t length = 0, T = 0, lmax = 127, stride = 1, pitch = 8;
  uint32_t* d_paths = nullptr;
  size_t paths_cap = 0;
  uint32_t* d_lengths = nullptr;
  size_t lengths_cap = 0;
  unsigned long long* d_visits = nullptr;  // [n] visit counts (cfg.visit_counts)
  size_t visits_cap = 0;
  uint32_t* d_visits32 = nullptr;          // [n] narrow counters (while counts fit in u32)
  size_t visits32_cap = 0;
  uint32_t* d_visits16 = nullptr;          // [ceil(n/2)] paired 16-bit counters (VIS 3)
  size_t visits16_cap = 0;
  unsigned long long* d_vsum = nullptr;    // [1] sum of the widened counts (VIS 3 wrap check)
  size_t vsum_cap = 0;
  uint32_t* d_slot = nullptr;              // [n] VIS 4 visit-count slot of each vertex (0: none), or nullptr
  size_t slot_cap = 0;
  uint32_t* d_vhot = nullptr;              // [kHotSlots] VIS 4 counters by slot
  size_t vhot_cap = 0;
  uint64_t hot_slots = 0;                  // slotted vertices (the highest degrees)
  uint4* d_vinfo = nullptr;                // [n] VIS 4 per-vertex {offset, slot, degree}
  size_t vinfo_cap = 0;
  bool visits_ready = false;
  uint32_t* d_starts = nullptr;
  size_t starts_cap = 0;
  uint32_t* d_starts_all = nullptr;  // lt_run_to_host*: every start, copied and validated once
  size_t starts_all_cap = 0;
  // walk admission (lt_config.walk_pool_walks): walks [0, admitted) have been created; at most
  // cap_walks are live; the rest are admitted from adm_starts as walks end
  const uint32_t* adm_starts = nullptr;
  uint64_t admitted = 0, cap_walks = 0;
  // pool
  uint4* d_slots = nullptr;
  size_t slots_cap = 0;
  uint32_t* d_ring = nullptr;
  size_t ring_cap = 0;
  unsigned long long* d_hc = nullptr;  // head[P] then cursor[P]
  size_t hc_cap = 0;
  uint32_t hs = 32;  // u64 per bucket block in d_hc (Pool::hs)
  uint32_t* d_free = nullptr;
  size_t free_cap = 0;
  uint32_t* d_small = nullptr;  // [0]=free_top [1]=unused [2..3]=scratch flags
  lt::Counters* d_ctr = nullptr;
  // pinned staging
  unsigned long long* h_hc = nullptr;  // mapped pinned: head[nb], cursor[nb]
  size_t h_hc_cap = 0;
  lt::Counters* h_ctr = nullptr;       // mapped pinned
  int* h_free = nullptr;               // mapped pinned: free-stack top
  lt::Params params{};
  lt_stats stats{};
  std::vector<cudaEvent_t> events;
  size_t nev = 0;
  // lt_run_to_host double buffers
  uint32_t* d_paths2[2] = {nullptr, nullptr};
  size_t paths2_cap[2] = {0, 0};
  uint32_t* d_lengths2[2] = {nullptr, nullptr};
  size_t lengths2_cap[2] = {0, 0};
  uint32_t* d_dense2[2] = {nullptr, nullptr};  // dense (stride-pitched) staging for the flat D2H
  size_t dense2_cap[2] = {0, 0};
  // compact (ragged) path output scratch: tile sums, total, offsets and packed vertices (x2 buffers)
  unsigned long long* d_tiles = nullptr;
  size_t tiles_cap = 0;
  unsigned long long* h_total = nullptr;  // mapped pinned
  unsigned long long* d_off2[2] = {nullptr, nullptr};
  size_t off2_cap[2] = {0, 0};
  uint32_t* d_vert2[2] = {nullptr, nullptr};
  size_t vert2_cap[2] = {0, 0};
  cudaStream_t copy_stream = nullptr;
  cudaEvent_t ev_computed[2] = {nullptr, nullptr}, ev_copied[2] = {nullptr, nullptr};
  cudaEvent_t ev_a = nullptr, ev_b = nullptr;
  // peer exchange (lt_exchange_buffers / lt_exchange_attach): this rank's two receive buffers and
  // cursors (epoch 0 / 1), and the device tables of every rank's buffers and cursors
  uint4* d_xbuf[2] = {nullptr, nullptr};
  unsigned long long* d_xcur = nullptr;  // [2]
  uint64_t xcap = 0;
  uint4** d_peer_recv = nullptr;                // [2 * world]
  unsigned long long** d_peer_cur = nullptr;    // [2 * world]
  bool peer_on = false;
  uint32_t peer_epoch = 0;
  std::vector<void*> ipc_opened;                // peer buffers opened through CUDA IPC (closed at destroy)
};

#define CK(call)                                                                        \
  do {                                                                                  \
    cudaError_t _e = (call);                                                            \
    if (_e != cudaSuccess)                                                              \
      return lt::fail(_e == cudaErrorMemoryAllocation ? LT_ERR_OOM : LT_ERR_CUDA,       \
                      std::string(#call) + ": " + cudaGetErrorString(_e));              \
  } while (0)

namespace lt {
lt_status snapshot(lt_ctx* ctx);  // h_hc / h_ctr / h_free <- device, then sync the stream
lt_status snapshot_cached(lt_ctx* ctx);  // snapshot() unless the mirror is still valid
lt_status run_resident(lt_ctx* ctx);
lt_status run_out_of_core(lt_ctx* ctx);
lt_status launch_update_timed(lt_ctx* ctx, const Params& p, uint32_t k, uint64_t walks_bound);
// admit walks while live < cap_walks (returns true in *did if any were admitted)
lt_status admit_walks(lt_ctx* ctx, uint64_t live, bool* did);
// walk spill: create every remaining walk, evicting chunks as the pool fills (lt_run's first step)
lt_status spill_admit_all(lt_ctx* ctx);
void free_spill(lt_ctx* ctx);
}  // namespace lt
