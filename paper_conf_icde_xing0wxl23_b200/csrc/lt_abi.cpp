// lt_abi.cpp — the C ABI (include/lt.h): context, validation, range partitioner (a1), graph
// loading (resident or out-of-core), pool reservation (a6 sizing) and outputs. The partition
// scheduler (a7; Alg. 2) is in lt_sched.cpp.
#include "lt_ctx.h"

#include <algorithm>
#include <cmath>
#include <atomic>
#include <thread>
#include <cstdio>
#include <cstring>
#include <numeric>
#include <string>
#include <vector>

namespace {
thread_local std::string g_err;
constexpr uint64_t kXcurStride = 32;  // u64 between the two exchange-epoch cursors (256 B)
}  // namespace

namespace lt {
lt_status fail(lt_status s, const std::string& msg) {
  g_err = msg;
  return s;
}

cudaError_t dmalloc(lt_ctx* ctx, void** p, size_t bytes) {
  if (!ctx->arena) return cudaMalloc(p, bytes);
  const size_t at = (ctx->arena_top + 255) & ~size_t(255);
  if (at + bytes > ctx->arena_size) return cudaErrorMemoryAllocation;  // -> LT_ERR_OOM
  *p = ctx->arena + at;
  ctx->arena_top = at + bytes;
  ctx->arena_peak = std::max(ctx->arena_peak, ctx->arena_top);
  return cudaSuccess;
}

void dfree(lt_ctx* ctx, void* p) {
  if (!p) return;
  if (ctx->arena && (char*)p >= ctx->arena && (char*)p < ctx->arena + ctx->arena_size) return;  // caller-owned
  cudaFree(p);
}

void arena_track(lt_ctx* ctx, void** p, size_t* cap) {
  if (!ctx->arena) return;
  for (const auto& b : ctx->arena_bufs)
    if (b.first == p) return;
  ctx->arena_bufs.emplace_back(p, cap);
}

// A graph load starts the arena over (every pool buffer is reserved again, graph first): the buffers of
// the previous graph and walks are dropped.
static void arena_reset(lt_ctx* ctx) {
  if (!ctx->arena) return;
  for (const auto& b : ctx->arena_bufs) {
    *b.first = nullptr;
    *b.second = 0;
  }
  for (int i = 0; i < 2; ++i) {
    ctx->d_paths2[i] = nullptr;
    ctx->paths2_cap[i] = 0;
    ctx->d_lengths2[i] = nullptr;
    ctx->lengths2_cap[i] = 0;
  }
  if (ctx->own_graph) {
    ctx->d_row_ptr = nullptr;
    ctx->d_col = nullptr;
  }
  ctx->d_owner = nullptr;
  ctx->walks_ready = false;
  ctx->arena_top = ctx->arena_mark;
}
}  // namespace lt
using lt::fail;
using lt::ensure;
using lt::dfree;
using lt::dmalloc;

extern "C" {

const char* lt_last_error(void) { return g_err.c_str(); }

lt_status lt_config_default(lt_config* cfg) {
  if (!cfg) return fail(LT_ERR_INVALID, "cfg is NULL");
  std::memset(cfg, 0, sizeof(*cfg));
  cfg->chunk_walks = 8192;
  cfg->ppr_max_len = 127;
  cfg->gather_mode = 3;
  return LT_OK;
}

lt_status lt_create(const lt_config* cfg, lt_ctx** out) {
  if (!out) return fail(LT_ERR_INVALID, "out is NULL");
  *out = nullptr;
  lt_config c;
  if (cfg) c = *cfg; else lt_config_default(&c);
  if (c.chunk_walks == 0) c.chunk_walks = 8192;
  if (c.chunk_walks < 64 || (c.chunk_walks & (c.chunk_walks - 1)))
    return fail(LT_ERR_INVALID, "chunk_walks must be a power of two >= 64");
  if (c.ppr_max_len == 0) c.ppr_max_len = 127;
  if (c.block_threads == 0) c.block_threads = 256;
  if (c.block_threads != 256) return fail(LT_ERR_INVALID, "block_threads must be 256 in this build");
  if (c.policy > 3 || c.insert_mode > 1 || c.gather_mode > 3 || c.zero_copy > 1)
    return fail(LT_ERR_INVALID, "bad policy / insert_mode / gather_mode");
  if (c.layout > 3) return fail(LT_ERR_INVALID, "bad layout");
  if (c.world == 0) c.world = 1;
  if (c.rank >= c.world || c.world > 65535) return fail(LT_ERR_INVALID, "need rank < world <= 65535");
  if (c.path_mode > 2) return fail(LT_ERR_INVALID, "bad path_mode");
  if (c.refill > 2) return fail(LT_ERR_INVALID, "bad refill");
  if (c.visit_counts > 2) return fail(LT_ERR_INVALID, "visit_counts must be 0, 1 or 2");
  if (c.direct_start > 1) return fail(LT_ERR_INVALID, "direct_start must be 0 (auto) or 1 (off)");
  if (c.ooc_compress > 1) return fail(LT_ERR_INVALID, "ooc_compress must be 0 (auto) or 1 (off)");
  if (c.walk_spill > 1) return fail(LT_ERR_INVALID, "walk_spill must be 0 or 1");
  if (c.ilp != 0 && c.ilp != 1 && c.ilp != 2 && c.ilp != 4) return fail(LT_ERR_INVALID, "ilp must be 0, 1, 2 or 4");
  int ndev = 0;
  CK(cudaGetDeviceCount(&ndev));
  if (c.device < 0 || c.device >= ndev) return fail(LT_ERR_INVALID, "bad device ordinal");
  CK(cudaSetDevice(c.device));
  lt_ctx* ctx = new lt_ctx();
  ctx->cfg = c;
  ctx->stream = (cudaStream_t)c.stream;
  ctx->block = c.block_threads;
  ctx->rank = c.rank;
  ctx->world = c.world;
  cudaDeviceGetAttribute(&ctx->num_sms, cudaDevAttrMultiProcessorCount, c.device);
  ctx->occ = 0;  // resolved per launch configuration in lt_walks_init
  // Every gather on the path touches one random 32-B sector; a larger L2 fetch granularity only
  // drags in neighbouring sectors nobody reads (measured: 2.5x DRAM read amplification at 64 B+).
  if (c.l2_fetch_bytes != 0xFFFFFFFFu) {
    size_t g = c.l2_fetch_bytes ? c.l2_fetch_bytes : 32;
    CK(cudaDeviceSetLimit(cudaLimitMaxL2FetchGranularity, g));
  }
  if (c.l2_persist > 1) {
    lt_destroy(ctx);
    return fail(LT_ERR_INVALID, "l2_persist must be 0 or 1");
  }
  cudaError_t e = cudaSuccess;
  if (c.l2_persist == 1) {  // evict_last lines (visit counters, row_ptr) get an L2 set-aside to stay in
    int mx = 0;
    size_t got = 0;
    e = cudaDeviceGetAttribute(&mx, cudaDevAttrMaxPersistingL2CacheSize, c.device);
    if (e == cudaSuccess && mx > 0) e = cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, (size_t)mx);
    if (e == cudaSuccess) e = cudaDeviceGetLimit(&got, cudaLimitPersistingL2CacheSize);
    ctx->stats.l2_persist_bytes = got;
  }
  if (c.arena || c.arena_bytes) {  // caller-owned device memory for every pool
    cudaPointerAttributes a{};
    if (!c.arena || c.arena_bytes < 4096 || cudaPointerGetAttributes(&a, c.arena) != cudaSuccess ||
        a.type != cudaMemoryTypeDevice || a.device != c.device) {
      (void)cudaGetLastError();
      lt_destroy(ctx);
      return fail(LT_ERR_INVALID, "arena must be device memory of cfg->device, >= 4096 bytes");
    }
    ctx->arena = (char*)c.arena;
    ctx->arena_size = c.arena_bytes;
  }
  if (e == cudaSuccess) e = dmalloc(ctx, (void**)&ctx->d_small, 4 * sizeof(uint32_t));
  if (e == cudaSuccess) e = dmalloc(ctx, (void**)&ctx->d_ctr, sizeof(lt::Counters));
  ctx->arena_mark = ctx->arena_top;
  if (e == cudaSuccess) e = cudaHostAlloc((void**)&ctx->h_ctr, sizeof(lt::Counters), cudaHostAllocMapped);
  if (e == cudaSuccess) e = cudaHostAlloc((void**)&ctx->h_free, sizeof(int), cudaHostAllocMapped);
  if (e == cudaSuccess) e = cudaEventCreate(&ctx->ev_a);
  if (e == cudaSuccess) e = cudaEventCreate(&ctx->ev_b);
  if (e != cudaSuccess) {
    lt_destroy(ctx);
    return fail(LT_ERR_CUDA, std::string("lt_create: ") + cudaGetErrorString(e));
  }
  *out = ctx;
  return LT_OK;
}

static void free_ooc(lt_ctx* ctx) {
  lt::OutOfCore& o = ctx->ooc;
  if (o.load_stream) cudaStreamSynchronize(o.load_stream);
  for (auto e : o.ev_ready) cudaEventDestroy(e);
  for (auto e : o.ev_used) cudaEventDestroy(e);
  if (o.load_stream) cudaStreamDestroy(o.load_stream);
  if (o.d_gpool) dfree(ctx, o.d_gpool);
  if (o.d_table) dfree(ctx, o.d_table);
  if (o.h_row_ptr) cudaFreeHost(o.h_row_ptr);
  if (o.h_col) cudaFreeHost(o.h_col);
  if (o.h_chdr) cudaFreeHost(o.h_chdr);
  if (o.h_cpay) cudaFreeHost(o.h_cpay);
  if (o.d_cstage) dfree(ctx, o.d_cstage);
  ctx->ooc = lt::OutOfCore();
}

void lt_destroy(lt_ctx* ctx) {
  if (!ctx) return;
  cudaSetDevice(ctx->cfg.device);
  if (ctx->stream) cudaStreamSynchronize(ctx->stream); else cudaDeviceSynchronize();
  free_ooc(ctx);
  lt::free_spill(ctx);
  ctx->load_ev.destroy();
  ctx->xfer_ev.destroy();
  if (ctx->own_graph) { dfree(ctx, ctx->d_row_ptr); dfree(ctx, ctx->d_col); }
  dfree(ctx, ctx->d_adj);
  dfree(ctx, ctx->d_adj12);
  dfree(ctx, ctx->d_bounds);
  dfree(ctx, ctx->d_owner);
  dfree(ctx, ctx->d_paths);
  dfree(ctx, ctx->d_lengths);
  for (int i = 0; i < 2; ++i) {
    if (ctx->d_paths2[i] && ctx->d_paths2[i] != ctx->d_paths) dfree(ctx, ctx->d_paths2[i]);
    if (ctx->d_lengths2[i] && ctx->d_lengths2[i] != ctx->d_lengths) dfree(ctx, ctx->d_lengths2[i]);
    if (ctx->d_dense2[i]) dfree(ctx, ctx->d_dense2[i]);
    if (ctx->d_off2[i]) dfree(ctx, ctx->d_off2[i]);
    if (ctx->d_vert2[i]) dfree(ctx, ctx->d_vert2[i]);
    if (ctx->ev_computed[i]) cudaEventDestroy(ctx->ev_computed[i]);
    if (ctx->ev_copied[i]) cudaEventDestroy(ctx->ev_copied[i]);
  }
  if (ctx->copy_stream) cudaStreamDestroy(ctx->copy_stream);
  for (void* q : ctx->ipc_opened) cudaIpcCloseMemHandle(q);
  cudaFree(ctx->d_xbuf[0]);
  cudaFree(ctx->d_xbuf[1]);
  cudaFree(ctx->d_xcur);
  cudaFree(ctx->d_peer_recv);
  cudaFree(ctx->d_peer_cur);
  dfree(ctx, ctx->d_starts);
  dfree(ctx, ctx->d_starts_all);
  dfree(ctx, ctx->d_visits);
  dfree(ctx, ctx->d_visits32);
  dfree(ctx, ctx->d_visits16);
  dfree(ctx, ctx->d_slot);
  dfree(ctx, ctx->d_vinfo);
  dfree(ctx, ctx->d_vhot);
  dfree(ctx, ctx->d_vsum);
  dfree(ctx, ctx->d_slots);
  dfree(ctx, ctx->d_ring);
  dfree(ctx, ctx->d_hc);
  dfree(ctx, ctx->d_free);
  dfree(ctx, ctx->d_small);
  dfree(ctx, ctx->d_tiles);
  if (ctx->h_total) cudaFreeHost(ctx->h_total);
  dfree(ctx, ctx->d_ctr);
  if (ctx->h_hc) cudaFreeHost(ctx->h_hc);
  if (ctx->h_ctr) cudaFreeHost(ctx->h_ctr);
  if (ctx->h_free) cudaFreeHost(ctx->h_free);
  for (auto ev : ctx->events) cudaEventDestroy(ev);
  if (ctx->ev_a) cudaEventDestroy(ctx->ev_a);
  if (ctx->ev_b) cudaEventDestroy(ctx->ev_b);
  delete ctx;
}

// a1: byte-balanced range partitioning, cost(v) = 8 v + 4 row_ptr[v] (the CSR prefix
// of vertices < v), bounds[k] = min{v : P cost(v) >= k cost(n)}, then made strictly increasing.
lt_status lt_partition_bounds(uint32_t n, const uint64_t* row_ptr, uint32_t P, uint32_t* bounds) {
  if (!row_ptr || !bounds) return fail(LT_ERR_INVALID, "NULL argument");
  if (P == 0 || P > n) return fail(LT_ERR_INVALID, "need 1 <= num_partitions <= n");
  auto cost = [&](uint64_t v) -> unsigned __int128 { return (unsigned __int128)8 * v + (unsigned __int128)4 * row_ptr[v]; };
  const unsigned __int128 total = cost(n);
  bounds[0] = 0;
  bounds[P] = n;
  for (uint32_t k = 1; k < P; ++k) {
    const unsigned __int128 target = total * k;
    uint64_t lo = 0, hi = n;  // first v with P cost(v) >= k cost(n)
    while (lo < hi) {
      const uint64_t mid = (lo + hi) / 2;
      if (cost(mid) * P < target) lo = mid + 1; else hi = mid;
    }
    bounds[k] = (uint32_t)lo;
  }
  for (uint32_t k = 1; k < P; ++k) bounds[k] = std::max(bounds[k], bounds[k - 1] + 1);
  for (uint32_t k = P - 1; k >= 1; --k) bounds[k] = std::min(bounds[k], bounds[k + 1] - 1);
  return LT_OK;
}

static lt_status validate_row_ptr(uint32_t n, uint64_t m, const uint64_t* row_ptr) {
  if (n == 0) return fail(LT_ERR_INVALID, "n must be >= 1");
  if (row_ptr[0] != 0) return fail(LT_ERR_INVALID, "row_ptr[0] != 0");
  if (row_ptr[n] != m) return fail(LT_ERR_INVALID, "row_ptr[n] != m");
  for (uint32_t v = 0; v < n; ++v) {
    if (row_ptr[v + 1] < row_ptr[v]) return fail(LT_ERR_INVALID, "row_ptr not monotone at " + std::to_string(v));
    if (row_ptr[v + 1] - row_ptr[v] > 0xFFFFFFFFull) return fail(LT_ERR_INVALID, "degree >= 2^32");
  }
  return LT_OK;
}

// Slice-only graph with range ownership ("each rank holds only its CSR slice"): the CSR
// entries of the vertices rank r owns, [row_ptr[b[own_lo]], row_ptr[b[own_hi]]). A step only ever
// gathers from the adjacency of an owned vertex: a walk that reaches another rank's vertex is sent
// there before its next step. The whole row_ptr stays (8 B per vertex): the ADJ build needs deg(u) and
// row_ptr[u] of every neighbour u, owned or not.
static lt_status owned_edges(lt_ctx* ctx, uint32_t n, uint64_t m, const uint64_t* h_row_ptr, uint32_t P, uint64_t* e_lo,
                             uint64_t* e_hi) {
  *e_lo = 0;
  *e_hi = m;
  const uint32_t R = ctx->world;
  if (R <= 1) return LT_OK;
  if (R > P) return fail(LT_ERR_INVALID, "need num_partitions >= world");
  std::vector<uint32_t> b(P + 1);
  lt_status s = lt_partition_bounds(n, h_row_ptr, P, b.data());
  if (s != LT_OK) return s;
  *e_lo = h_row_ptr[b[(uint64_t)P * ctx->rank / R]];
  *e_hi = h_row_ptr[b[(uint64_t)P * (ctx->rank + 1) / R]];
  return LT_OK;
}

static lt_status finish_graph_load(lt_ctx* ctx, uint32_t n, uint64_t m, const uint64_t* h_row_ptr, uint32_t P) {
  CK(cudaEventRecord(ctx->ev_a, ctx->stream));
  // Layout: the augmented adjacency costs 16 B per CSR entry and saves one
  // random DRAM access per step; auto-select it when it fits in half of the free device memory.
  // (with ownership only the owned slice [e_lo, e_hi) is built)
  // The compact 12-B form (LT_LAYOUT_ADJ12) packs row_ptr[u] into 40 bits and deg(u) into 24: it is
  // taken when asked for, or by auto when only 12 B per entry fit.
  const uint64_t ml = ctx->ooc.on ? m : ctx->e_hi - ctx->e_lo;
  uint64_t dmax = 0;
  for (uint32_t v = 0; v < n; ++v) dmax = std::max<uint64_t>(dmax, h_row_ptr[v + 1] - h_row_ptr[v]);
  const bool fits12 = m < (1ull << 40) && dmax < (1ull << 24);
  int lay = LT_LAYOUT_CSR;
  if (!ctx->ooc.on && ml) {
    if (ctx->cfg.layout == LT_LAYOUT_ADJ) {
      if (m >= (1ull << 40)) return fail(LT_ERR_INVALID, "LT_LAYOUT_ADJ needs m < 2^40 (40-bit offsets)");
      lay = LT_LAYOUT_ADJ;
    }
    if (ctx->cfg.layout == LT_LAYOUT_ADJ12) {
      if (!fits12) return fail(LT_ERR_INVALID, "LT_LAYOUT_ADJ12 needs m < 2^40 and every degree < 2^24");
      lay = LT_LAYOUT_ADJ12;
    }
    if (ctx->cfg.layout == LT_LAYOUT_AUTO) {
      // Measured on B200 (profiles/r01_gather_tlb_reach.json): random gathers run at the full access
      // rate over up to 64 GiB and fall off beyond it (72 GiB 0.87x, 80 GiB 0.62x, 128 GiB 0.27x), the
      // reach of the GPU's address translation. An augmented array past that reach loses more than the
      // row_ptr access it saves, so it is only chosen within it.
      constexpr double kGatherReach = 64.0 * (1ull << 30);
      size_t fr = 0, tot = 0;
      CK(cudaMemGetInfo(&fr, &tot));
      // an augmented array this context already holds is replaced (or reused) by this load: count it as free
      if (!ctx->cfg.arena) fr += ctx->adj_cap * sizeof(uint4) + ctx->adj12_cap * 4;
      const double a16 = (double)ml * 16.0, a12 = (double)ml * 12.0;
      if (a16 <= 0.5 * (double)fr && a16 <= kGatherReach && m < (1ull << 40)) lay = LT_LAYOUT_ADJ;
      else if (fits12 && a12 <= 0.5 * (double)fr && a12 <= kGatherReach) lay = LT_LAYOUT_ADJ12;
    }
  }
  // VIS 4 slots (visit counting on, one rank, ADJ): the kHotSlots - 1 highest-degree vertices get slots 1..,
  // in descending degree order (a counting sort of the degrees), embedded in the ADJ entries below
  ctx->hot_slots = 0;
  if (lay == LT_LAYOUT_ADJ && ctx->cfg.visit_counts == 1 && ctx->world == 1 && ctx->cfg.gather_mode == 3 && n) {
    std::vector<uint64_t> cnt(dmax + 2, 0);
    for (uint32_t v = 0; v < n; ++v) cnt[h_row_ptr[v + 1] - h_row_ptr[v]]++;
    // start of each degree's ranks in descending order
    std::vector<uint64_t> at(dmax + 2, 0);
    uint64_t acc = 0;
    for (uint64_t dg = dmax + 1; dg-- > 0;) {
      at[dg] = acc;
      acc += cnt[dg];
    }
    std::vector<uint32_t> slot(n);
    for (uint32_t v = 0; v < n; ++v) {
      const uint64_t r = at[h_row_ptr[v + 1] - h_row_ptr[v]]++;
      slot[v] = r + 1 < lt::kHotSlots ? (uint32_t)(r + 1) : 0u;
    }
    ctx->hot_slots = std::min<uint64_t>(n, lt::kHotSlots - 1);
    CK(ensure(ctx, ctx->d_slot, ctx->slot_cap, n));
    CK(cudaMemcpyAsync(ctx->d_slot, slot.data(), (size_t)n * 4, cudaMemcpyHostToDevice, ctx->stream));
    CK(ensure(ctx, ctx->d_vinfo, ctx->vinfo_cap, n));
    CK(lt::launch_build_vinfo(ctx->d_row_ptr, ctx->d_slot, n, ctx->d_vinfo, ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
  }
  if (lay == LT_LAYOUT_ADJ) {
    CK(ensure(ctx, ctx->d_adj, ctx->adj_cap, ml));
    CK(lt::launch_build_adj(ctx->d_row_ptr, ctx->d_col, ml, ctx->d_adj, ctx->hot_slots ? ctx->d_slot : nullptr,
                            ctx->stream));
  } else if (ctx->d_adj) {
    dfree(ctx, ctx->d_adj);
    ctx->d_adj = nullptr;
    ctx->adj_cap = 0;
  }
  if (lay == LT_LAYOUT_ADJ12) {
    CK(ensure(ctx, ctx->d_adj12, ctx->adj12_cap, 3 * ml));
    CK(lt::launch_build_adj12(ctx->d_row_ptr, ctx->d_col, ml, ctx->d_adj12, ctx->stream));
  } else if (ctx->d_adj12) {
    dfree(ctx, ctx->d_adj12);
    ctx->d_adj12 = nullptr;
    ctx->adj12_cap = 0;
  }
  // the steps of an augmented layout never read col: a col the library owns is released (a borrowed
  // one may be released by the caller, include/lt.h)
  if (lay != LT_LAYOUT_CSR && ctx->own_graph && ctx->d_col) {
    CK(cudaStreamSynchronize(ctx->stream));
    dfree(ctx, ctx->d_col);
    ctx->d_col = nullptr;
  }
  ctx->stats.layout = (uint32_t)lay;
  ctx->stats.graph_device_bytes = ctx->ooc.on ? 0
      : ((uint64_t)n + 1) * 8 + ml * (lay == LT_LAYOUT_ADJ ? 16 : lay == LT_LAYOUT_ADJ12 ? 12 : 4);
  ctx->stats.out_of_core = ctx->ooc.on ? 1 : 0;
  std::vector<uint32_t> b(P + 1);
  lt_status s = lt_partition_bounds(n, h_row_ptr, P, b.data());
  if (s != LT_OK) return s;
  CK(ensure(ctx, ctx->d_bounds, ctx->bounds_cap, P + 1));
  CK(cudaMemcpy(ctx->d_bounds, b.data(), (P + 1) * sizeof(uint32_t), cudaMemcpyHostToDevice));
  // range ownership: rank r owns partitions [floor(P r / R), floor(P (r+1) / R))
  const uint32_t R = ctx->world;
  if (R > P) return fail(LT_ERR_INVALID, "need num_partitions >= world");
  ctx->own_lo = (uint32_t)((uint64_t)P * ctx->rank / R);
  ctx->own_hi = (uint32_t)((uint64_t)P * (ctx->rank + 1) / R);
  ctx->nb = P + (R > 1 ? R : 0);
  if (ctx->d_owner) dfree(ctx, ctx->d_owner);
  ctx->d_owner = nullptr;
  if (R > 1) {
    std::vector<uint16_t> own(P);
    for (uint32_t r = 0; r < R; ++r)
      for (uint64_t q = (uint64_t)P * r / R; q < (uint64_t)P * (r + 1) / R; ++q) own[q] = (uint16_t)r;
    CK(dmalloc(ctx, (void**)&ctx->d_owner, P * sizeof(uint16_t)));
    CK(cudaMemcpy(ctx->d_owner, own.data(), P * sizeof(uint16_t), cudaMemcpyHostToDevice));
  }
  const size_t nb = ctx->nb;
  // head, cursor, refill claim of bucket b in block b of hs u64 (Pool::hs): 256 B per bucket while there
  // are few buckets (each insertion cursor on its own L2 line), 32 B beyond
  ctx->hs = nb <= 4096 ? 32 : 4;
  CK(ensure(ctx, ctx->d_hc, ctx->hc_cap, ctx->hs * nb));
  if (ctx->h_hc_cap < 2 * nb) {
    if (ctx->h_hc) cudaFreeHost(ctx->h_hc);
    ctx->h_hc = nullptr;
    ctx->h_hc_cap = 0;
    CK(cudaHostAlloc((void**)&ctx->h_hc, 2 * nb * sizeof(unsigned long long), cudaHostAllocMapped));
    ctx->h_hc_cap = 2 * nb;
  }
  CK(cudaEventRecord(ctx->ev_b, ctx->stream));
  CK(cudaEventSynchronize(ctx->ev_b));
  {
    float ms = 0;
    CK(cudaEventElapsedTime(&ms, ctx->ev_a, ctx->ev_b));
    ctx->stats.graph_prep_ms = ms;
  }
  ctx->h_bounds = std::move(b);
  ctx->n = n;
  ctx->m = m;
  ctx->P = P;
  ctx->graph_loaded = true;
  ctx->walks_ready = false;
  ctx->ran = false;
  return LT_OK;
}

// Compressed partition transfers (lt_config.ooc_compress): each partition's column slice is
// cut into blocks of 32 entries; block j stores its first value and the zigzag-coded differences of
// consecutive entries (mod 2^32, so any values round-trip), bit-packed at the block's width w (the bits of
// the largest code) in exactly w payload words. Sorted adjacency lists give small differences, so the
// link carries fewer bytes; a partition whose blocks would not be smaller than its raw slice travels raw.
// Host threads build it once per lt_graph_load* (two passes: widths, then packing).
static inline uint32_t zz(uint32_t d) { return (d << 1) ^ (uint32_t)((int32_t)d >> 31); }

// width of block j of a slice (bits of its largest zigzag code; 0 when all entries are equal)
static inline uint32_t block_width(const uint32_t* c, uint64_t L) {
  uint32_t mx = 0;
  for (uint64_t i = 1; i < L; ++i) mx = std::max(mx, zz(c[i] - c[i - 1]));
  return mx ? (uint32_t)(32 - __builtin_clz(mx)) : 0u;
}

// encode blocks [0, nblk) of a slice of len entries into hdr[nblk + 1] / pay (payload words zeroed here)
static void encode_slice(const uint32_t* col, uint64_t len, const uint8_t* width, uint2* hdr, uint32_t* pay) {
  const uint64_t nblk = (len + 31) / 32;
  uint64_t off = 0;
  for (uint64_t j = 0; j < nblk; ++j) {
    const uint32_t* c = col + 32 * j;
    const uint64_t L = std::min<uint64_t>(32, len - 32 * j);
    const uint32_t w = width[j];
    hdr[j] = make_uint2(c[0], (uint32_t)off);
    for (uint32_t q = 0; q < w; ++q) pay[off + q] = 0;
    for (uint64_t i = 1; i < L && w; ++i) {
      const uint64_t z = zz(c[i] - c[i - 1]), bit = i * w;
      pay[off + (bit >> 5)] |= (uint32_t)(z << (bit & 31));
      if ((bit & 31) + w > 32) pay[off + (bit >> 5) + 1] |= (uint32_t)(z >> (32 - (bit & 31)));
    }
    off += w;
  }
  hdr[nblk] = make_uint2(0, (uint32_t)off);  // sentinel: the last block's width
}

static lt_status compress_columns(lt_ctx* ctx, const std::vector<uint32_t>& b, uint32_t P) {
  lt::OutOfCore& o = ctx->ooc;
  std::vector<uint64_t> nblk(P), words(P, 0);
  std::vector<std::vector<uint8_t>> width(P);
  std::atomic<uint32_t> next{0};
  auto pass1 = [&]() {
    for (uint32_t k; (k = next.fetch_add(1)) < P;) {
      const uint64_t e0 = o.h_row_ptr[b[k]], e1 = o.h_row_ptr[b[k + 1]], len = e1 - e0;
      nblk[k] = (len + 31) / 32;
      width[k].resize(nblk[k]);
      uint64_t wsum = 0;
      for (uint64_t j = 0; j < nblk[k]; ++j) {
        width[k][j] = (uint8_t)block_width(o.h_col + e0 + 32 * j, std::min<uint64_t>(32, len - 32 * j));
        wsum += width[k][j];
      }
      words[k] = wsum;
    }
  };
  const unsigned nt = std::max(1u, std::min(16u, std::thread::hardware_concurrency()));
  {
    std::vector<std::thread> th;
    for (unsigned t = 0; t < nt; ++t) th.emplace_back(pass1);
    for (auto& x : th) x.join();
  }
  o.craw.assign(P, 0);
  o.chdr_at.assign(P + 1, 0);
  o.cpay_at.assign(P + 1, 0);
  uint64_t stage = 0;
  for (uint32_t k = 0; k < P; ++k) {
    const uint64_t raw = 4ull * (o.h_row_ptr[b[k + 1]] - o.h_row_ptr[b[k]]);
    const uint64_t comp = 8ull * (nblk[k] + 1) + 4ull * words[k];
    if (words[k] >= 0xFFFFFFFFull || comp >= raw) {
      o.craw[k] = 1;
      nblk[k] = 0;
      words[k] = 0;
    } else {
      stage = std::max<uint64_t>(stage, comp);
    }
    o.chdr_at[k + 1] = o.chdr_at[k] + (o.craw[k] ? 0 : nblk[k] + 1);
    o.cpay_at[k + 1] = o.cpay_at[k] + words[k];
  }
  if (!stage) return LT_OK;  // nothing shrinks: raw copies only
  // the blocks are an optimisation: without the pinned host memory for them, partitions travel raw
  if (cudaHostAlloc((void**)&o.h_chdr, o.chdr_at[P] * sizeof(uint2), cudaHostAllocPortable) != cudaSuccess ||
      cudaHostAlloc((void**)&o.h_cpay, std::max<uint64_t>(o.cpay_at[P], 1) * 4, cudaHostAllocPortable) != cudaSuccess) {
    (void)cudaGetLastError();
    if (o.h_chdr) cudaFreeHost(o.h_chdr);
    o.h_chdr = nullptr;
    o.h_cpay = nullptr;
    o.craw.assign(P, 1);
    return LT_OK;
  }
  next = 0;
  auto pass2 = [&]() {
    for (uint32_t k; (k = next.fetch_add(1)) < P;) {
      if (o.craw[k]) continue;
      const uint64_t e0 = o.h_row_ptr[b[k]], len = o.h_row_ptr[b[k + 1]] - e0;
      encode_slice(o.h_col + e0, len, width[k].data(), o.h_chdr + o.chdr_at[k], o.h_cpay + o.cpay_at[k]);
    }
  };
  {
    std::vector<std::thread> th;
    for (unsigned t = 0; t < nt; ++t) th.emplace_back(pass2);
    for (auto& x : th) x.join();
  }
  o.cstage_bytes = (stage + 255) & ~255ull;
  CK(dmalloc(ctx, (void**)&o.d_cstage, o.cstage_bytes));
  o.comp = true;
  o.comp_bytes = 8ull * o.chdr_at[P] + 4ull * o.cpay_at[P];
  return LT_OK;
}

// Out-of-core graph (a7/a8): G_cpu is a pinned, mapped host copy of the CSR;
// the device graph pool holds m_g blocks, each big enough for the largest partition's row_ptr slice
// (at offset 0) plus col slice (at rp_bytes).
static lt_status setup_out_of_core(lt_ctx* ctx, uint32_t n, uint64_t m, const uint64_t* row_ptr, const uint32_t* col,
                                   bool src_on_device, uint32_t P) {
  free_ooc(ctx);
  lt::OutOfCore& o = ctx->ooc;
  CK(cudaHostAlloc((void**)&o.h_row_ptr, ((size_t)n + 1) * 8, cudaHostAllocMapped | cudaHostAllocPortable));
  CK(cudaHostAlloc((void**)&o.h_col, std::max<uint64_t>(m, 1) * 4, cudaHostAllocMapped | cudaHostAllocPortable));
  if (src_on_device) {
    CK(cudaMemcpy(o.h_row_ptr, row_ptr, ((size_t)n + 1) * 8, cudaMemcpyDeviceToHost));
    if (m) CK(cudaMemcpy(o.h_col, col, m * 4, cudaMemcpyDeviceToHost));
  } else {
    std::memcpy(o.h_row_ptr, row_ptr, ((size_t)n + 1) * 8);
    const unsigned nt = 8;
    std::vector<std::thread> th;
    for (unsigned t = 0; t < nt; ++t)
      th.emplace_back([&, t] {
        const uint64_t a = m * t / nt, b = m * (t + 1) / nt;
        if (b > a) std::memcpy(o.h_col + a, col + a, (b - a) * 4);
      });
    for (auto& x : th) x.join();
  }
  CK(cudaHostGetDevicePointer((void**)&o.d_map_row_ptr, o.h_row_ptr, 0));
  CK(cudaHostGetDevicePointer((void**)&o.d_map_col, o.h_col, 0));
  std::vector<uint32_t> b(P + 1);
  lt_status s = lt_partition_bounds(n, (const uint64_t*)o.h_row_ptr, P, b.data());
  if (s != LT_OK) return s;
  uint64_t rp_max = 0, col_max = 0;
  for (uint32_t k = 0; k < P; ++k) {
    rp_max = std::max<uint64_t>(rp_max, 8ull * (b[k + 1] - b[k] + 1));
    col_max = std::max<uint64_t>(col_max, 4ull * (o.h_row_ptr[b[k + 1]] - o.h_row_ptr[b[k]]));
  }
  o.rp_bytes = (rp_max + 255) & ~255ull;
  o.block_bytes = (o.rp_bytes + col_max + 255) & ~255ull;
  if (ctx->cfg.ooc_compress == 0 && m) {
    lt_status cs = compress_columns(ctx, b, P);
    if (cs != LT_OK) return cs;
  }
  uint64_t mg = ctx->cfg.graph_pool_bytes / o.block_bytes;
  if (mg == 0)
    return fail(LT_ERR_INVALID, "graph pool smaller than one partition (" + std::to_string(o.block_bytes) +
                                    " B): raise num_partitions or graph_pool_bytes");
  o.m_g = (uint32_t)std::min<uint64_t>(mg, P);
  CK(dmalloc(ctx, (void**)&o.d_gpool, (size_t)o.m_g * o.block_bytes));
  o.block_of.assign(P, -1);
  o.part_in.assign(o.m_g, -1);
  o.loaded_at.assign(o.m_g, 0);
  o.ev_ready.resize(o.m_g);
  o.ev_used.resize(o.m_g);
  for (uint32_t q = 0; q < o.m_g; ++q) {
    CK(cudaEventCreateWithFlags(&o.ev_ready[q], cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&o.ev_used[q], cudaEventDisableTiming));
  }
  CK(cudaStreamCreateWithFlags(&o.load_stream, cudaStreamNonBlocking));
  CK(dmalloc(ctx, (void**)&o.d_table, (size_t)P * sizeof(uint32_t)));
  CK(cudaMemset(o.d_table, 0xFF, (size_t)P * sizeof(uint32_t)));
  o.table.assign(P, lt::kEmpty);
  o.on = true;
  ctx->stats.pool_blocks = o.m_g;
  ctx->stats.pool_block_bytes = o.block_bytes;
  ctx->stats.ooc_compressed_bytes = o.comp_bytes;
  return LT_OK;
}

lt_status lt_graph_load(lt_ctx* ctx, uint32_t n, uint64_t m, const uint64_t* row_ptr, const uint32_t* col,
                        uint32_t P) {
  if (!ctx || !row_ptr || (m && !col)) return fail(LT_ERR_INVALID, "NULL argument");
  CK(cudaSetDevice(ctx->cfg.device));
  lt_status s = validate_row_ptr(n, m, row_ptr);
  if (s != LT_OK) return s;
  for (uint64_t i = 0; i < m; ++i)
    if (col[i] >= n) return fail(LT_ERR_INVALID, "col[" + std::to_string(i) + "] >= n");
  if (P == 0 || P > n) return fail(LT_ERR_INVALID, "need 1 <= num_partitions <= n");
  CK(cudaDeviceSynchronize());  // nothing in flight reads the buffers the load replaces
  if (ctx->own_graph) { dfree(ctx, ctx->d_row_ptr); dfree(ctx, ctx->d_col); }
  lt::arena_reset(ctx);
  ctx->d_row_ptr = nullptr;
  ctx->d_col = nullptr;
  ctx->graph_loaded = false;
  free_ooc(ctx);
  if (ctx->cfg.graph_pool_bytes) {
    ctx->own_graph = false;
    ctx->e_lo = 0;
    ctx->e_hi = m;
    lt_status so = setup_out_of_core(ctx, n, m, row_ptr, col, false, P);
    if (so != LT_OK) return so;
    return finish_graph_load(ctx, n, m, row_ptr, P);
  }
  uint64_t e_lo = 0, e_hi = m;
  s = owned_edges(ctx, n, m, row_ptr, P, &e_lo, &e_hi);
  if (s != LT_OK) return s;
  ctx->own_graph = true;
  CK(dmalloc(ctx, (void**)&ctx->d_row_ptr, ((size_t)n + 1) * sizeof(uint64_t)));
  CK(dmalloc(ctx, (void**)&ctx->d_col, std::max<uint64_t>(e_hi - e_lo, 1) * sizeof(uint32_t)));
  CK(cudaMemcpy(ctx->d_row_ptr, row_ptr, ((size_t)n + 1) * sizeof(uint64_t), cudaMemcpyHostToDevice));
  if (e_hi > e_lo) CK(cudaMemcpy(ctx->d_col, col + e_lo, (e_hi - e_lo) * sizeof(uint32_t), cudaMemcpyHostToDevice));
  ctx->e_lo = e_lo;
  ctx->e_hi = e_hi;
  ctx->stats.h2d_bytes += ((uint64_t)n + 1) * 8 + (e_hi - e_lo) * 4;
  return finish_graph_load(ctx, n, m, row_ptr, P);
}

lt_status lt_graph_load_device(lt_ctx* ctx, uint32_t n, uint64_t m, const uint64_t* d_row_ptr, const uint32_t* d_col,
                               uint32_t P) {
  if (!ctx || !d_row_ptr || (m && !d_col)) return fail(LT_ERR_INVALID, "NULL argument");
  CK(cudaSetDevice(ctx->cfg.device));
  std::vector<uint64_t> h((size_t)n + 1);
  CK(cudaMemcpy(h.data(), d_row_ptr, ((size_t)n + 1) * sizeof(uint64_t), cudaMemcpyDeviceToHost));
  lt_status s = validate_row_ptr(n, m, h.data());
  if (s != LT_OK) return s;
  if (P == 0 || P > n) return fail(LT_ERR_INVALID, "need 1 <= num_partitions <= n");
  CK(cudaMemsetAsync(ctx->d_small + 2, 0, sizeof(uint32_t), ctx->stream));
  CK(lt::launch_check_col(d_col, m, n, ctx->d_small + 2, ctx->stream));
  uint32_t bad = 0;
  CK(cudaMemcpyAsync(&bad, ctx->d_small + 2, sizeof(uint32_t), cudaMemcpyDeviceToHost, ctx->stream));
  CK(cudaStreamSynchronize(ctx->stream));
  if (bad) return fail(LT_ERR_INVALID, "col entry >= n");
  CK(cudaDeviceSynchronize());
  if (ctx->own_graph) { dfree(ctx, ctx->d_row_ptr); dfree(ctx, ctx->d_col); }
  lt::arena_reset(ctx);
  ctx->own_graph = false;
  ctx->graph_loaded = false;
  free_ooc(ctx);
  if (ctx->cfg.graph_pool_bytes) {  // host-resident copy of the caller's device CSR
    ctx->d_row_ptr = nullptr;
    ctx->d_col = nullptr;
    ctx->e_lo = 0;
    ctx->e_hi = m;
    lt_status so = setup_out_of_core(ctx, n, m, d_row_ptr, d_col, true, P);
    if (so != LT_OK) return so;
    return finish_graph_load(ctx, n, m, h.data(), P);
  }
  uint64_t e_lo = 0, e_hi = m;
  s = owned_edges(ctx, n, m, h.data(), P, &e_lo, &e_hi);
  if (s != LT_OK) return s;
  ctx->d_row_ptr = (unsigned long long*)d_row_ptr;
  ctx->d_col = (uint32_t*)d_col + e_lo;  // a view of the owned slice of the caller's array
  ctx->e_lo = e_lo;
  ctx->e_hi = e_hi;
  return finish_graph_load(ctx, n, m, h.data(), P);
}

lt_status lt_get_bounds(lt_ctx* ctx, uint32_t* bounds, uint32_t* P) {
  if (!ctx) return fail(LT_ERR_INVALID, "NULL ctx");
  if (!ctx->graph_loaded) return fail(LT_ERR_STATE, "no graph loaded");
  if (P) *P = ctx->P;
  if (bounds) std::memcpy(bounds, ctx->h_bounds.data(), (ctx->P + 1) * sizeof(uint32_t));
  return LT_OK;
}

lt_status lt_walks_init(lt_ctx* ctx, uint64_t W, const uint32_t* starts, lt_app app, double param, uint64_t seed) {
  return lt_walks_init_ex(ctx, W, starts, 0, 0, app, param, seed);
}

static lt_status walks_init_impl(lt_ctx* ctx, uint64_t W, const uint32_t* starts, int on_device,
                                 uint64_t first_walk_id, lt_app app, double length_d, double alpha, uint64_t seed);

lt_status lt_walks_init_ex(lt_ctx* ctx, uint64_t W, const uint32_t* starts, int on_device, uint64_t first_walk_id,
                           lt_app app, double param, uint64_t seed) {
  if (app == LT_APP_PAGERANK) return fail(LT_ERR_INVALID, "PageRank takes a length and p: use lt_walks_init_pagerank");
  on_device = on_device ? 1 : 0;
  if (app == LT_APP_DEEPWALK) return walks_init_impl(ctx, W, starts, on_device, first_walk_id, app, param, 0.0, seed);
  return walks_init_impl(ctx, W, starts, on_device, first_walk_id, app, 0.0, param, seed);
}

lt_status lt_walks_init_pagerank(lt_ctx* ctx, uint64_t W, const uint32_t* starts, int on_device,
                                 uint64_t first_walk_id, uint32_t length, double restart_p, uint64_t seed) {
  return walks_init_impl(ctx, W, starts, on_device ? 1 : 0, first_walk_id, LT_APP_PAGERANK, (double)length, restart_p,
                         seed);
}

static lt_status walks_init_impl(lt_ctx* ctx, uint64_t W, const uint32_t* starts, int on_device,
                                 uint64_t first_walk_id, lt_app app, double length_d, double alpha, uint64_t seed) {
  if (!ctx) return fail(LT_ERR_INVALID, "NULL ctx");
  lt::Range rg("lt_walks_init");
  if (!ctx->graph_loaded) return fail(LT_ERR_STATE, "lt_walks_init before lt_graph_load");
  if (W && !starts) return fail(LT_ERR_INVALID, "starts is NULL");
  if (W >= 0xFFFFFFFFull) return fail(LT_ERR_INVALID, "num_walks must be < 2^32 - 1");
  CK(cudaSetDevice(ctx->cfg.device));
  uint32_t length = 0, T = 0, stride = 0;
  const uint32_t lmax = ctx->cfg.ppr_max_len;
  if (app == LT_APP_DEEPWALK || app == LT_APP_PAGERANK) {
    if (!(length_d >= 0) || length_d != std::floor(length_d) || length_d > 1e6)
      return fail(LT_ERR_INVALID, "walk length must be an integer in [0, 1e6]");
    length = (uint32_t)length_d;
    stride = length + 1;
  }
  if (app == LT_APP_PPR || app == LT_APP_PAGERANK) {
    if (!(alpha > 0 && alpha < 1))
      return fail(LT_ERR_INVALID, "PPR alpha / PageRank restart probability must be in (0, 1)");
    const double t = alpha * 4294967296.0;  // T = floor(alpha 2^32) (reading R5)
    T = (uint32_t)t;
    if (app == LT_APP_PPR) stride = lmax + 1;
  } else if (app != LT_APP_DEEPWALK) {
    return fail(LT_ERR_INVALID, "unknown app");
  }
  if (ctx->cfg.walk_pool_walks && ctx->world != 1)
    return fail(LT_ERR_INVALID, "walk_pool_walks (walk admission) needs a single-rank context");
  ctx->walks_ready = false;
  ctx->visits_ready = false;
  ctx->ran = false;
  ctx->stats.h2d_bytes = 0;
  ctx->stats.d2h_bytes = 0;
  cudaStream_t s = ctx->stream;
  // starts (on_device: 1 = caller's device array, validated below; 2 = internal, already validated)
  const uint32_t* d_starts = starts;
  if (!on_device) {
    for (uint64_t i = 0; i < W; ++i)
      if (starts[i] >= ctx->n) return fail(LT_ERR_INVALID, "starts[" + std::to_string(i) + "] >= n");
    CK(ensure(ctx, ctx->d_starts, ctx->starts_cap, W));
    if (W) CK(cudaMemcpyAsync(ctx->d_starts, starts, W * sizeof(uint32_t), cudaMemcpyHostToDevice, s));
    ctx->stats.h2d_bytes += W * 4;
    d_starts = ctx->d_starts;
  }
  // reserve: paths, lengths, pool
  const uint64_t C = ctx->cfg.chunk_walks;
  uint32_t c_shift = 0;
  while ((1ull << c_shift) < C) ++c_shift;
  // walk pool: sized for the walks that can be live at once
  const uint64_t cap = (ctx->cfg.walk_pool_walks && ctx->cfg.walk_pool_walks < W) ? ctx->cfg.walk_pool_walks : W;
  // direct start (lt_config.direct_start): with one partition every new walk belongs to bucket 0, so
  // the lane-refill kernel (the P == 1 default) takes walk j straight from starts[j]: k_init (16-B
  // record write + read back + one bucket cursor atomic per warp) is skipped and, since a walk never
  // leaves the only partition, no record is ever appended: the pool keeps only its per-bucket slack
  const bool direct = ctx->cfg.direct_start == 0 && (ctx->cfg.refill == 0 || ctx->cfg.refill == 2) && ctx->P == 1 &&
                      ctx->world == 1 && !ctx->ooc.on && cap == W;
  const uint64_t wc = direct ? 0 : (cap + C - 1) / C;
  // A bucket spans at most wc + 2 chunks, except with continuation during a zero-copy launch of
  // partition i: a walk that goes i -> resident q -> i finds no block for i and is appended to bucket i
  // while that launch still consumes [head, tail), so the bucket can span twice the walks.
  const bool reenter = ctx->ooc.on && ctx->cfg.continue_resident && ctx->cfg.zero_copy;
  // with walk spill a bucket's positions [head, cursor) may hold every walk (evicted chunks keep their
  // ring slots), so its ring spans all W walks, not just the pool's
  const bool spill = ctx->cfg.walk_spill == 1 && cap < W;
  const uint64_t wr = spill ? (W + C - 1) / C : wc;
  const uint64_t ring_len = reenter ? 2 * wr + 3 : wr + 2;
  const uint64_t num_chunks = 2 * wc + 2 * (uint64_t)ctx->nb + 64;
  if (num_chunks >= 0x7FFFFFFFull) return fail(LT_ERR_INVALID, "pool too large; raise chunk_walks");
  const uint32_t pitch = (stride + 7u) & ~7u;  // rows start on 32-B sectors
  // path_mode 2 stores no path entries (the paper's accounting): no path matrix. A rank
  // whose paths go to a home rank (lt_paths_attach) keeps no matrix of its own either.
  const bool home = ctx->home_paths != nullptr && ctx->world > 1 && ctx->cfg.path_mode != 2;
  if (home && (uint64_t)W * pitch > ctx->home_cap)
    return fail(LT_ERR_INVALID, "the home rank's path matrix is smaller than W x pitch; attach again");
  CK(ensure(ctx, ctx->d_paths, ctx->paths_cap, (ctx->cfg.path_mode == 2 || home) ? 8 : std::max<uint64_t>(W, 1) * pitch));
  CK(ensure(ctx, ctx->d_lengths, ctx->lengths_cap, std::max<uint64_t>(W, 1)));
  CK(ensure(ctx, ctx->d_slots, ctx->slots_cap, (num_chunks + 1) * C));
  CK(ensure(ctx, ctx->d_ring, ctx->ring_cap, (uint64_t)ctx->nb * ring_len));
  CK(ensure(ctx, ctx->d_free, ctx->free_cap, num_chunks));
  // visit counters: u32 while no count can reach 2^32 (at most W * stride path entries in total)
  const bool narrow = ctx->cfg.visit_counts == 1 && (uint64_t)W * stride < 0xFFFFFFFFull;
  if (ctx->cfg.visit_counts) CK(ensure(ctx, ctx->d_visits, ctx->visits_cap, ctx->n));
  if (narrow) CK(ensure(ctx, ctx->d_visits32, ctx->visits32_cap, ctx->n));
  // Paired 16-bit counters for the non-hub vertices (VIS 3, DESIGN.md §7 "PageRank and visit counts"):
  // with an augmented layout (the step knows the visited vertex's degree), one rank, the graph resident.
  // A hub is a vertex whose expected count could approach 2^16: with Nt = W * stride path entries at most
  // and the walk's arrival rate at v about deg(v) / m per step (+ alpha / n per step for restarts, + the
  // starts), deg >= hub_deg keeps every non-hub's expected count <= 4096 (16x below the wrap). A wrap is
  // still possible (e.g. all starts on one low-degree vertex); it is detected exactly and recounted.
  uint32_t hub_deg = 0;
  bool half = false;
  // VIS 4 (counters by degree slot) when the ADJ entries carry slots; else VIS 3 below
  const bool slots = narrow && ctx->hot_slots && ctx->d_adj && ctx->world == 1 && !ctx->ooc.on;
  if (slots) {
    CK(ensure(ctx, ctx->d_vhot, ctx->vhot_cap, lt::hot_index((uint32_t)ctx->hot_slots) + 1));
  }
  if (!slots && narrow && ctx->world == 1 && !ctx->ooc.on && (ctx->d_adj || ctx->d_adj12) && ctx->cfg.gather_mode == 3 &&
      ctx->m && W) {
    const double Nt = (double)W * stride;
    const double rest = (app == LT_APP_PAGERANK ? Nt * alpha : 0.0) / ctx->n + (double)W / ctx->n;
    const double h = (4096.0 - rest) * (double)ctx->m / Nt;
    if (h >= 64.0) {
      half = true;
      hub_deg = h > 4e9 ? 0xFFFFFFFFu : (uint32_t)h;
    }
  }
  if (half) {
    CK(ensure(ctx, ctx->d_visits16, ctx->visits16_cap, (ctx->n + 1) / 2));
    CK(ensure(ctx, ctx->d_vsum, ctx->vsum_cap, 1));
  }
  if (on_device == 1 && W) {
    CK(cudaMemsetAsync(ctx->d_small + 2, 0, sizeof(uint32_t), s));
    CK(lt::launch_check_starts(d_starts, W, ctx->n, ctx->d_small + 2, s));
    uint32_t bad = 0;
    CK(cudaMemcpyAsync(&bad, ctx->d_small + 2, sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    if (bad) return fail(LT_ERR_INVALID, "a start vertex >= n");
  }
  lt::Params& p = ctx->params;
  p.wk.row_ptr = ctx->d_row_ptr;
  p.wk.col = ctx->d_col;
  p.wk.vbase = 0;
  p.wk.ebase = ctx->ooc.on ? 0 : ctx->e_lo;  // col / adj hold the CSR entries from e_lo on (ownership slice)
  p.wk.adj = ctx->ooc.on ? nullptr : ctx->d_adj;
  p.wk.adj12 = ctx->ooc.on ? nullptr : ctx->d_adj12;
  p.wk.bounds = ctx->d_bounds;
  p.wk.P = ctx->P;
  p.wk.paths = home ? ctx->home_paths : ctx->d_paths;
  p.sys_fence = home ? 1u : 0u;
  p.wk.stride = stride;
  p.wk.pitch = pitch;
  p.wk.path_mode = ctx->cfg.path_mode;
  p.wk.lengths = home ? ctx->home_lengths : ctx->d_lengths;
  p.wk.first_walk_id = first_walk_id;
  p.wk.seed_lo = (uint32_t)seed;
  p.wk.seed_hi = (uint32_t)(seed >> 32);
  p.wk.app = (uint32_t)app;
  p.wk.length = length;
  p.wk.T = T;
  p.wk.lmax = lmax;
  p.wk.n = ctx->n;
  p.wk.visits = ctx->cfg.visit_counts ? ctx->d_visits : nullptr;
  p.wk.visits32 = narrow ? ctx->d_visits32 : nullptr;
  p.wk.visits16 = half ? ctx->d_visits16 : nullptr;
  p.wk.vhot = slots ? ctx->d_vhot : nullptr;
  p.wk.vinfo = slots ? ctx->d_vinfo : nullptr;
  ctx->stats.visit_hot_slots = slots ? ctx->hot_slots : 0;
  p.wk.hub_deg = hub_deg;
  ctx->stats.hub_deg = hub_deg;
  ctx->stats.visit_recounts = 0;
  p.pool.slots = ctx->d_slots;
  p.pool.C = (uint32_t)C;
  p.pool.c_shift = c_shift;
  p.pool.num_chunks = (uint32_t)num_chunks;
  p.pool.ring = ctx->d_ring;
  p.pool.ring_len = (uint32_t)ring_len;
  p.pool.nbuckets = ctx->nb;
  p.pool.head = ctx->d_hc;
  p.pool.cursor = ctx->d_hc + 1;
  p.pool.claim = ctx->d_hc + 2;
  p.pool.hs = ctx->hs;
  p.own.own_lo = ctx->own_lo;
  p.own.own_hi = ctx->own_hi;
  p.own.owner = ctx->d_owner;
  p.pool.free_list = ctx->d_free;
  p.pool.free_top = (int*)ctx->d_small;
  p.ctr = ctx->d_ctr;
  p.cont = lt::Cont{};
  if (ctx->ooc.on && ctx->cfg.continue_resident)
    p.cont = lt::Cont{ctx->ooc.d_table, ctx->ooc.d_gpool, ctx->ooc.block_bytes, ctx->ooc.rp_bytes};
  p.tail_cap = ~0ull;
  p.insert_mode = ctx->cfg.insert_mode;
  p.gather_mode = ctx->cfg.gather_mode;
  // measured best: 1 walk per lane with the one-gather-per-step ADJ layout, 2 with CSR
  p.ilp = ctx->cfg.ilp ? ctx->cfg.ilp : ((p.wk.adj || p.wk.adj12) ? 1u : 2u);
  // lane refill (k_update_rf): measured faster with one partition (DeepWalk 65.5 vs 81.7 ms, PPR 6.2
  // vs 7.7 ms on cfg 4 / cfg 3); with O records (round 2) also at P = 4 (15.7 vs 14.2-14.4·10^9 steps/s
  // on cfg 4, four runs), P = 16 (8.7-8.8 vs 8.4-8.6, three runs), P = 8 in one of two runs (12.7 vs 12.2;
  // 11.1 vs 11.8), tied at P = 64 and behind at P = 256 (3.8 vs 4.0), DESIGN.md §8
  // (second session: with the sorted flush — at most 64 buckets, C >= 128, aggregated insertion — lane refill
  // also wins at P = 32 (11.8 vs 10.8) and P = 64 (9.8 vs 9.3), profiles/r02b_sorted_flush.txt)
  const bool sorted_flush = ctx->nb <= 64 && ctx->cfg.chunk_walks >= 128 && ctx->cfg.insert_mode == 0;
  p.refill = ctx->cfg.refill == 2 || (ctx->cfg.refill == 0 && (ctx->P <= 16 || sorted_flush)) ? 1u : 0u;
  if (p.cont.table) p.refill = 1;  // continuation lives in the lane-refill kernel
  if (p.refill) p.ilp = 1;
  ctx->occ = ctx->cfg.blocks_per_sm ? (int)ctx->cfg.blocks_per_sm
                                    : lt::update_kernel_occupancy(ctx->block, p.ilp, p.refill, p.wk.app, ctx->P);
  p.direct = direct ? lt::Direct{d_starts, W} : lt::Direct{nullptr, 0};
  p.peer = ctx->peer_on ? lt::Peer{ctx->d_peer_recv, ctx->d_peer_cur, ctx->xcap, ctx->peer_epoch} : lt::Peer{};
  ctx->stats.direct_start = direct ? 1 : 0;

  ctx->W = W;
  ctx->first = first_walk_id;
  ctx->seed = seed;
  ctx->app = app;
  ctx->length = length;
  ctx->T = T;
  ctx->lmax = lmax;
  ctx->stride = stride;
  ctx->pitch = pitch;
  ctx->stats.num_walks = W;
  ctx->stats.chunks_total = num_chunks;
  ctx->stats.kernel_launches = 0;
  // per-epoch statistics: with range ownership lt_run (and lt_superstep_p2p) is called once per
  // superstep and these accumulate over the epoch's supersteps, like the device step counter
  ctx->stats.sweeps = 0;
  ctx->stats.update_launches = 0;
  ctx->stats.update_ms = 0;
  ctx->stats.iterations = 0;
  ctx->stats.explicit_copies = 0;
  ctx->stats.pool_hits = 0;
  ctx->stats.zero_copy_launches = 0;
  ctx->stats.preemptive_launches = 0;
  ctx->stats.prefetches = 0;
  ctx->stats.graph_h2d_bytes = 0;
  ctx->stats.graph_h2d_raw_bytes = 0;
  ctx->stats.run_ms = 0;
  ctx->stats.chunks_free_min = num_chunks;
  ctx->stats.spilled_chunks = 0;
  ctx->stats.reloaded_chunks = 0;
  ctx->stats.spill_d2h_bytes = 0;
  ctx->stats.spill_h2d_bytes = 0;
  ctx->stats.host_chunks_peak = 0;
  ctx->stats.spill_prefetched_chunks = 0;
  ctx->stats.load_ms = 0;
  ctx->stats.spill_xfer_ms = 0;
  ctx->stats.host_syncs = 0;
  ctx->load_ev.n = 0;
  ctx->xfer_ev.n = 0;
  ctx->nev = 0;
  // walk spill (lt_config.walk_spill): every walk exists from lt_run's start; the pool of num_chunks
  // chunks evicts to a pinned host store of one slot per chunk the W walks can fill (+ partial chunks)
  {
    lt::Spill& sp = ctx->spill;
    sp.on = ctx->cfg.walk_spill == 1 && cap < W;
    if (sp.on) {
      const uint64_t host_cap = (W + C - 1) / C + ctx->nb + 2;
      if (sp.host_cap < host_cap) {
        CK(cudaStreamSynchronize(ctx->stream));
        if (sp.h_store) cudaFreeHost(sp.h_store);
        sp.h_store = nullptr;
        sp.d_store = nullptr;
        sp.host_cap = 0;
        CK(cudaHostAlloc((void**)&sp.h_store, host_cap * C * sizeof(uint4), cudaHostAllocPortable | cudaHostAllocMapped));
        CK(cudaHostGetDevicePointer((void**)&sp.d_store, sp.h_store, 0));
        sp.host_cap = host_cap;
      }
      sp.spilled.assign(ctx->nb, {});
      sp.host_free.resize(sp.host_cap);
      for (uint64_t i = 0; i < sp.host_cap; ++i) sp.host_free[i] = (uint32_t)(sp.host_cap - 1 - i);
      sp.host_used = 0;
      sp.free_chunks = (int64_t)num_chunks;
    }
  }
  CK(cudaEventRecord(ctx->ev_a, s));
  ctx->snap_valid = false;
  CK(lt::launch_pool_reset(p, s));
  ctx->stats.kernel_launches++;
  // The home rank's matrix and lengths are written by every rank without a per-epoch barrier: after the
  // first epoch it neither pre-fills nor zeroes them (every length is written once per epoch by the rank
  // where the walk ends; the rows are padded lazily by the first copy-out, R24).
  if (W && !home && !ctx->is_home) CK(cudaMemsetAsync(ctx->d_lengths, 0, W * sizeof(uint32_t), s));
  if (narrow) CK(cudaMemsetAsync(ctx->d_visits32, 0, (size_t)ctx->n * sizeof(uint32_t), s));
  if (half) CK(cudaMemsetAsync(ctx->d_visits16, 0, (size_t)((ctx->n + 1) / 2) * sizeof(uint32_t), s));
  if (slots) CK(cudaMemsetAsync(ctx->d_vhot, 0, (size_t)(lt::hot_index((uint32_t)ctx->hot_slots) + 1) * sizeof(uint32_t), s));
  else if (ctx->cfg.visit_counts) CK(cudaMemsetAsync(ctx->d_visits, 0, (size_t)ctx->n * sizeof(unsigned long long), s));
  // with range ownership each rank writes only its share of every row: unwritten entries must
  // read 0xFFFFFFFF so that the cross-rank merge is an element-wise min
  // (path_mode 2 stores no rows: d_paths is a placeholder of 8 entries and there is nothing to merge)
  if (W && ctx->world > 1 && ctx->cfg.path_mode != 2 && !home && !ctx->is_home)
    CK(cudaMemsetAsync(ctx->d_paths, 0xFF, W * (uint64_t)pitch * sizeof(uint32_t), s));
  ctx->adm_starts = d_starts;
  ctx->cap_walks = cap;
  ctx->admitted = cap;
  ctx->stats.admissions = 0;
  ctx->stats.peak_live = cap;
  if (cap) {
    if (!direct) {
      CK(lt::launch_init(p, d_starts, cap, 0, s));
      ctx->stats.kernel_launches++;
    }
    ctx->stats.admissions = 1;
  }
  CK(cudaEventRecord(ctx->ev_b, s));
  ctx->walks_ready = true;
  return LT_OK;
}

lt_status lt_run(lt_ctx* ctx) {
  if (!ctx) return fail(LT_ERR_INVALID, "NULL ctx");
  lt::Range rg("lt_run");
  if (!ctx->walks_ready) return fail(LT_ERR_STATE, "lt_run before lt_walks_init");
  if (ctx->ran && ctx->world == 1)
    return fail(LT_ERR_STATE, "lt_run already done for these walks; call lt_walks_init again");
  CK(cudaSetDevice(ctx->cfg.device));
  cudaStream_t s = ctx->stream;
  if (!ctx->ran) {
    float ms = 0;
    CK(cudaEventSynchronize(ctx->ev_b));
    CK(cudaEventElapsedTime(&ms, ctx->ev_a, ctx->ev_b));
    ctx->stats.init_ms = ms;
  }
  // (update launches recorded since the last lt_run — e.g. by lt_superstep_p2p — stay in events[0, nev)
  // and are summed below; the per-epoch counters were reset by lt_walks_init)
  CK(cudaEventRecord(ctx->ev_a, s));
  lt_status st = LT_OK;
  if (ctx->spill.on && !ctx->ran) st = lt::spill_admit_all(ctx);  // walk spill: every walk exists from here on
  if (st != LT_OK) return st;
  st = ctx->ooc.on ? lt::run_out_of_core(ctx) : lt::run_resident(ctx);
  if (st != LT_OK) return st;
  if (ctx->spill.on) {
    for (const auto& m : ctx->spill.spilled)
      if (!m.empty()) return fail(LT_ERR_CUDA, "walk spill: evicted chunks left behind (invariant violated)");
  }
  // Path rows hold entries 0..length-1; the 0xFFFFFFFF padding of the rest is output formatting and is
  // written lazily by the first copy-out (ensure_padded). With ownership the rows were pre-filled.
  ctx->padded = ctx->world > 1 && !ctx->is_home;
  if (ctx->params.wk.vhot) {  // the result is u64[n]: per-vertex counts plus the slotted ones
    CK(lt::launch_widen_slots(ctx->params.wk.visits32, ctx->params.wk.vhot, ctx->d_slot, ctx->params.wk.visits,
                              ctx->n, s));
    ctx->stats.kernel_launches++;
  } else if (ctx->params.wk.visits16) {  // the result is u64[n]; the sum of all counts checks for a 16-bit wrap
    CK(cudaMemsetAsync(ctx->d_vsum, 0, sizeof(unsigned long long), s));
    CK(lt::launch_widen16(ctx->params.wk.visits16, ctx->params.wk.visits32, ctx->d_row_ptr, ctx->params.wk.hub_deg,
                          ctx->params.wk.visits, ctx->n, ctx->d_vsum, s));
    ctx->stats.kernel_launches++;
  } else if (ctx->params.wk.visits32) {  // the result is u64[n]
    CK(lt::launch_widen(ctx->params.wk.visits32, ctx->params.wk.visits, ctx->n, s));
    ctx->stats.kernel_launches++;
  }
  CK(cudaEventRecord(ctx->ev_b, s));
  st = lt::snapshot_cached(ctx);  // the scheduler's last count read (nothing moved since) or a fresh one
  if (st != LT_OK) return st;
  CK(cudaEventSynchronize(ctx->ev_b));
  {
    float ms = 0;
    CK(cudaEventElapsedTime(&ms, ctx->ev_a, ctx->ev_b));
    ctx->stats.run_ms += ms;
    double tot = 0;
    for (size_t i = 0; i + 1 < ctx->nev; i += 2) {
      CK(cudaEventElapsedTime(&ms, ctx->events[i], ctx->events[i + 1]));
      tot += ms;
    }
    ctx->stats.update_ms += tot;
    ctx->nev = 0;
    double t = 0;
    if (ctx->ooc.load_stream) CK(cudaStreamSynchronize(ctx->ooc.load_stream));
    CK(ctx->load_ev.total_ms(&t));
    ctx->stats.load_ms += t;
    CK(ctx->xfer_ev.total_ms(&t));
    ctx->stats.spill_xfer_ms += t;
  }
  ctx->stats.steps = ctx->h_ctr->steps;
  ctx->stats.visits = ctx->h_ctr->visits;
  ctx->stats.truncated = ctx->h_ctr->truncated;
  if (ctx->params.wk.visits16) {
    // every walk has 1 + (its steps) path entries; a wrapped 16-bit half loses 2^16 (or 2^16 - 1 with the
    // carry into its neighbour) from the sum, so sum == entries iff nothing wrapped
    unsigned long long sum = 0;
    CK(cudaMemcpy(&sum, ctx->d_vsum, sizeof(sum), cudaMemcpyDeviceToHost));
    const unsigned long long entries = ctx->h_ctr->steps + ctx->W;
    ctx->stats.visit_recounts = 0;
    if (sum != entries) {
      if (ctx->cfg.path_mode == 2)
        return fail(LT_ERR_INVALID, "a 16-bit visit counter wrapped and path_mode 2 keeps no paths to recount "
                                    "from; set visit_counts = 2 (u64 counters)");
      CK(cudaMemsetAsync(ctx->params.wk.visits, 0, (size_t)ctx->n * sizeof(unsigned long long), s));
      CK(lt::launch_recount(ctx->params.wk.paths, ctx->params.wk.pitch, ctx->params.wk.lengths, ctx->W,
                            ctx->params.wk.visits, s));
      CK(cudaStreamSynchronize(s));
      ctx->stats.visit_recounts = 1;
    }
  }
  ctx->ran = true;
  ctx->visits_ready = ctx->cfg.visit_counts != 0;
  if (ctx->h_ctr->err & lt::kErrOOM) return fail(LT_ERR_CUDA, "walk pool exhausted on the device (invariant violated)");
  if (ctx->h_ctr->err & lt::kErrPeer)
    return fail(LT_ERR_INVALID, "a peer receive buffer overflowed; raise the lt_exchange_buffers capacity");
  if (ctx->h_ctr->err) return fail(LT_ERR_CUDA, "device invariant violated (ring slot reinstalled)");
  return LT_OK;
}

lt_status lt_path_stride(lt_ctx* ctx, uint32_t* stride) {
  if (!ctx || !stride) return fail(LT_ERR_INVALID, "NULL argument");
  if (!ctx->walks_ready) return fail(LT_ERR_STATE, "no walks");
  *stride = ctx->stride;
  return LT_OK;
}

static lt_status need_ran(lt_ctx* ctx) {
  if (!ctx) return fail(LT_ERR_INVALID, "NULL ctx");
  if (!ctx->ran) return fail(LT_ERR_STATE, "paths requested before lt_run");
  if (ctx->cfg.path_mode != 2 && ctx->params.wk.paths != ctx->d_paths)
    return fail(LT_ERR_STATE, "this rank's paths and lengths were written into the home rank's matrix "
                              "(lt_paths_attach): read them there");
  CK(cudaSetDevice(ctx->cfg.device));
  if (!ctx->padded && ctx->cfg.path_mode != 2) {  // pad unused path slots with 0xFFFFFFFF once, before the first copy-out
    CK(lt::launch_finalize_paths(ctx->params, ctx->W, ctx->stream));
    ctx->padded = true;
  }
  return LT_OK;
}

static lt_status need_paths(lt_ctx* ctx) {
  if (ctx->cfg.path_mode == 2) return fail(LT_ERR_STATE, "paths are not stored (path_mode 2)");
  if (ctx->params.wk.paths != ctx->d_paths)
    return fail(LT_ERR_STATE, "this rank's paths were written into the home rank's matrix (lt_paths_attach)");
  return LT_OK;
}

lt_status lt_get_paths(lt_ctx* ctx, uint32_t* paths, uint32_t* lengths) {
  lt_status st = need_ran(ctx);
  if (st != LT_OK) return st;
  if (paths && (st = need_paths(ctx)) != LT_OK) return st;
  CK(cudaSetDevice(ctx->cfg.device));
  cudaStream_t s = ctx->stream;
  if (paths && ctx->W) {
    CK(cudaMemcpy2DAsync(paths, ctx->stride * sizeof(uint32_t), ctx->d_paths, ctx->pitch * sizeof(uint32_t),
                         ctx->stride * sizeof(uint32_t), ctx->W, cudaMemcpyDeviceToHost, s));
    ctx->stats.d2h_bytes += ctx->W * ctx->stride * 4;
  }
  if (lengths && ctx->W) {
    CK(cudaMemcpyAsync(lengths, ctx->d_lengths, ctx->W * sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
    ctx->stats.d2h_bytes += ctx->W * 4;
  }
  CK(cudaStreamSynchronize(s));
  return LT_OK;
}

lt_status lt_get_paths_rows(lt_ctx* ctx, const uint64_t* rows, uint64_t count, uint32_t* paths, uint32_t* lengths) {
  lt_status st = need_ran(ctx);
  if (st != LT_OK) return st;
  if ((st = need_paths(ctx)) != LT_OK) return st;
  if (count && (!rows || !paths || !lengths)) return fail(LT_ERR_INVALID, "NULL argument");
  for (uint64_t i = 0; i < count; ++i)
    if (rows[i] >= ctx->W) return fail(LT_ERR_INVALID, "row index >= W");
  if (!count) return LT_OK;
  CK(cudaSetDevice(ctx->cfg.device));
  cudaStream_t s = ctx->stream;
  unsigned long long* d_rows = nullptr;
  uint32_t* d_out = nullptr;
  uint32_t* d_len = nullptr;
  CK(cudaMalloc((void**)&d_rows, count * sizeof(uint64_t)));
  cudaError_t e = cudaMalloc((void**)&d_out, count * ctx->stride * sizeof(uint32_t));
  if (e == cudaSuccess) e = cudaMalloc((void**)&d_len, count * sizeof(uint32_t));
  if (e == cudaSuccess) e = cudaMemcpyAsync(d_rows, rows, count * sizeof(uint64_t), cudaMemcpyHostToDevice, s);
  if (e == cudaSuccess) e = lt::launch_gather_rows(ctx->params, d_rows, count, d_out, d_len, s);
  if (e == cudaSuccess) e = cudaMemcpyAsync(paths, d_out, count * ctx->stride * sizeof(uint32_t), cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess) e = cudaMemcpyAsync(lengths, d_len, count * sizeof(uint32_t), cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  cudaFree(d_rows);
  cudaFree(d_out);
  cudaFree(d_len);
  if (e != cudaSuccess) return fail(LT_ERR_CUDA, std::string("lt_get_paths_rows: ") + cudaGetErrorString(e));
  return LT_OK;
}

lt_status lt_get_paths_device(lt_ctx* ctx, uint32_t* d_paths, uint32_t* d_lengths) {
  lt_status st = need_ran(ctx);
  if (st != LT_OK) return st;
  if (d_paths && (st = need_paths(ctx)) != LT_OK) return st;
  CK(cudaSetDevice(ctx->cfg.device));
  cudaStream_t s = ctx->stream;
  if (d_paths && ctx->W)
    CK(cudaMemcpy2DAsync(d_paths, ctx->stride * sizeof(uint32_t), ctx->d_paths, ctx->pitch * sizeof(uint32_t),
                         ctx->stride * sizeof(uint32_t), ctx->W, cudaMemcpyDeviceToDevice, s));
  if (d_lengths && ctx->W)
    CK(cudaMemcpyAsync(d_lengths, ctx->d_lengths, ctx->W * sizeof(uint32_t), cudaMemcpyDeviceToDevice, s));
  CK(cudaStreamSynchronize(s));
  return LT_OK;
}

// Pack rows [0, n) of (paths, lengths) into buffer b: offsets (n entries, base + exclusive prefix sum)
// and vertices; returns the range's vertex total (synchronises the stream once, for the total).
static lt_status pack_compact(lt_ctx* ctx, const uint32_t* d_paths, const uint32_t* d_lengths, uint64_t n, int b,
                              unsigned long long base, uint64_t* total) {
  cudaStream_t s = ctx->stream;
  if (!ctx->h_total) CK(cudaHostAlloc((void**)&ctx->h_total, sizeof(unsigned long long), cudaHostAllocMapped));
  unsigned long long* d_total = nullptr;
  CK(cudaHostGetDevicePointer((void**)&d_total, ctx->h_total, 0));
  CK(ensure(ctx, ctx->d_tiles, ctx->tiles_cap, std::max<uint64_t>(lt::paths_scan_tiles(n), 1)));
  CK(ensure(ctx, ctx->d_off2[b], ctx->off2_cap[b], std::max<uint64_t>(n, 1)));
  *ctx->h_total = 0;
  CK(lt::launch_paths_scan(d_lengths, n, ctx->d_tiles, d_total, s));
  CK(cudaStreamSynchronize(s));
  const uint64_t tot = *(volatile unsigned long long*)ctx->h_total;
  CK(ensure(ctx, ctx->d_vert2[b], ctx->vert2_cap[b], std::max<uint64_t>(tot, 1)));
  CK(lt::launch_paths_pack(d_lengths, n, ctx->d_tiles, base, ctx->d_off2[b], d_paths, ctx->pitch, ctx->d_vert2[b], s));
  *total = tot;
  return LT_OK;
}

lt_status lt_get_paths_compact(lt_ctx* ctx, uint64_t* offsets, uint32_t* vertices, uint64_t vertices_capacity,
                               uint64_t* total) {
  if (!ctx || !offsets || !total) return fail(LT_ERR_INVALID, "NULL argument");
  if (!ctx->ran) return fail(LT_ERR_STATE, "paths requested before lt_run");
  if (need_paths(ctx) != LT_OK) return LT_ERR_STATE;
  CK(cudaSetDevice(ctx->cfg.device));
  uint64_t tot = 0;
  lt_status st = pack_compact(ctx, ctx->d_paths, ctx->d_lengths, ctx->W, 0, 0, &tot);
  if (st != LT_OK) return st;
  cudaStream_t s = ctx->stream;
  if (ctx->W) CK(cudaMemcpyAsync(offsets, ctx->d_off2[0], ctx->W * sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
  offsets[ctx->W] = tot;
  *total = tot;
  if (tot > vertices_capacity) {
    CK(cudaStreamSynchronize(s));
    return fail(LT_ERR_INVALID, "vertices buffer too small: need " + std::to_string(tot));
  }
  if (tot && !vertices) return fail(LT_ERR_INVALID, "NULL vertices");
  if (tot) CK(cudaMemcpyAsync(vertices, ctx->d_vert2[0], tot * sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
  ctx->stats.d2h_bytes += ctx->W * 8 + tot * 4;
  CK(cudaStreamSynchronize(s));
  return LT_OK;
}

lt_status lt_get_pool_state(lt_ctx* ctx, lt_pool_state* out) {
  if (!ctx || !out) return fail(LT_ERR_INVALID, "NULL argument");
  if (!ctx->walks_ready) return fail(LT_ERR_STATE, "no walks");
  CK(cudaSetDevice(ctx->cfg.device));
  CK(cudaStreamSynchronize(ctx->stream));
  const lt::Params& p = ctx->params;
  std::memset(out, 0, sizeof(*out));
  int32_t small[2] = {0, 0};
  CK(cudaMemcpy(small, ctx->d_small, sizeof(small), cudaMemcpyDeviceToHost));
  lt::Counters c;
  CK(cudaMemcpy(&c, ctx->d_ctr, sizeof(c), cudaMemcpyDeviceToHost));
  std::vector<uint32_t> ring((size_t)ctx->nb * p.pool.ring_len);
  CK(cudaMemcpy(ring.data(), ctx->d_ring, ring.size() * sizeof(uint32_t), cudaMemcpyDeviceToHost));
  std::vector<unsigned long long> hcs((size_t)ctx->nb * ctx->hs), hc(2 * (size_t)ctx->nb);
  CK(cudaMemcpy(hcs.data(), ctx->d_hc, hcs.size() * sizeof(unsigned long long), cudaMemcpyDeviceToHost));
  for (size_t b = 0; b < ctx->nb; ++b) {
    hc[b] = hcs[b * ctx->hs];
    hc[ctx->nb + b] = hcs[b * ctx->hs + 1];
  }
  std::vector<uint32_t> len(ctx->W);
  if (ctx->W) CK(cudaMemcpy(len.data(), ctx->d_lengths, ctx->W * sizeof(uint32_t), cudaMemcpyDeviceToHost));
  out->free_chunks = small[0];
  out->total_chunks = p.pool.num_chunks;
  for (uint32_t r : ring) {
    out->ring_chunks += (r != lt::kEmpty && r != lt::kSpilled);
    out->host_chunks += (r == lt::kSpilled);
  }
  for (uint32_t k = 0; k < ctx->nb; ++k) out->pending += hc[ctx->nb + k] - hc[k];
  if (ctx->ran) out->finished = ctx->W;  // every walk terminated
  else for (uint32_t l : len) out->finished += (l != 0 && l != lt::kEmpty);
  out->device_err = c.err;
  return LT_OK;
}

lt_status lt_pending(lt_ctx* ctx, uint64_t* local, uint64_t* outgoing) {
  if (!ctx) return fail(LT_ERR_INVALID, "NULL ctx");
  if (!ctx->walks_ready) return fail(LT_ERR_STATE, "no walks");
  CK(cudaSetDevice(ctx->cfg.device));
  const size_t nb = ctx->nb;
  lt_status sn = lt::snapshot_cached(ctx);
  if (sn != LT_OK) return sn;
  uint64_t loc = 0;
  for (uint32_t k = ctx->own_lo; k < ctx->own_hi; ++k) loc += ctx->h_hc[nb + k] - ctx->h_hc[k];
  if (local) *local = loc;
  if (outgoing)
    for (uint32_t r = 0; r < ctx->world; ++r)
      outgoing[r] = ctx->world > 1 ? ctx->h_hc[nb + ctx->P + r] - ctx->h_hc[ctx->P + r] : 0;
  return LT_OK;
}

lt_status lt_exchange_pack(lt_ctx* ctx, void* d_send, uint64_t capacity, uint64_t* counts) {
  if (!ctx || !counts) return fail(LT_ERR_INVALID, "NULL argument");
  if (!ctx->walks_ready) return fail(LT_ERR_STATE, "no walks");
  std::vector<uint64_t> out(ctx->world, 0);
  lt_status st = lt_pending(ctx, nullptr, out.data());
  if (st != LT_OK) return st;
  uint64_t total = 0;
  for (uint64_t c : out) total += c;
  if (total > capacity) return fail(LT_ERR_INVALID, "send buffer too small: need " + std::to_string(total));
  if (total && !d_send) return fail(LT_ERR_INVALID, "NULL send buffer");
  uint64_t off = 0;
  for (uint32_t r = 0; r < ctx->world; ++r) {
    counts[r] = out[r];
    if (!out[r]) continue;
    ctx->snap_valid = false;
    CK(lt::launch_pack(ctx->params, ctx->P + r, (uint4*)d_send + off, out[r], ctx->stream));
    ctx->stats.kernel_launches++;
    off += out[r];
  }
  // no host synchronisation: the buffer is complete in stream order, which is what the collective that
  // sends it (enqueued after this call on the same stream) needs
  return LT_OK;
}

lt_status lt_exchange_insert(lt_ctx* ctx, const void* d_recv, uint64_t count) {
  if (!ctx) return fail(LT_ERR_INVALID, "NULL ctx");
  if (!ctx->walks_ready) return fail(LT_ERR_STATE, "no walks");
  if (count && !d_recv) return fail(LT_ERR_INVALID, "NULL receive buffer");
  if (count) ctx->snap_valid = false;
  CK(lt::launch_insert_records(ctx->params, (const uint4*)d_recv, count, ctx->stream));
  if (count) ctx->stats.kernel_launches++;
  return LT_OK;  // stream-ordered: the next lt_run's first count read synchronises
}

// ---- peer exchange (walks appended straight into the owner's receive buffer over peer memory)
lt_status lt_exchange_buffers(lt_ctx* ctx, uint64_t capacity, void** recv, void** cursor) {
  if (!ctx || !recv || !cursor) return fail(LT_ERR_INVALID, "NULL argument");
  if (ctx->world < 2) return fail(LT_ERR_INVALID, "lt_exchange_buffers needs world > 1");
  if (!capacity) return fail(LT_ERR_INVALID, "capacity must be > 0");
  CK(cudaSetDevice(ctx->cfg.device));
  if (ctx->xcap != capacity) {
    if (ctx->peer_on) return fail(LT_ERR_STATE, "peer buffers are attached; their capacity is fixed");
    for (int e = 0; e < 2; ++e) {
      cudaFree(ctx->d_xbuf[e]);
      ctx->d_xbuf[e] = nullptr;
      CK(cudaMalloc(&ctx->d_xbuf[e], capacity * sizeof(uint4)));
    }
    // the two epochs' cursors (every sender's append atomic lands on one of them) in separate 256-B blocks
    if (!ctx->d_xcur) CK(cudaMalloc(&ctx->d_xcur, 2 * kXcurStride * sizeof(unsigned long long)));
    CK(cudaMemset(ctx->d_xcur, 0, 2 * kXcurStride * sizeof(unsigned long long)));
    ctx->xcap = capacity;
  }
  for (int e = 0; e < 2; ++e) {
    recv[e] = ctx->d_xbuf[e];
    cursor[e] = ctx->d_xcur + e * kXcurStride;
  }
  return LT_OK;
}

lt_status lt_exchange_attach(lt_ctx* ctx, void* const* recv, void* const* cursor) {
  if (!ctx || !recv || !cursor) return fail(LT_ERR_INVALID, "NULL argument");
  if (!ctx->xcap) return fail(LT_ERR_STATE, "lt_exchange_attach before lt_exchange_buffers");
  const uint32_t R = ctx->world;
  for (uint32_t i = 0; i < 2 * R; ++i)
    if (!recv[i] || !cursor[i]) return fail(LT_ERR_INVALID, "NULL peer buffer or cursor");
  if (recv[ctx->rank] != ctx->d_xbuf[0] || recv[R + ctx->rank] != ctx->d_xbuf[1])
    return fail(LT_ERR_INVALID, "the table's entry for this rank must be this rank's own buffers");
  CK(cudaSetDevice(ctx->cfg.device));
  // Peer buffers on another device of this process (threads driving several GPUs): the update kernels'
  // atomics and stores into them need peer access from this context's device (IPC-opened buffers
  // already map with cudaIpcMemLazyEnablePeerAccess).
  for (uint32_t i = 0; i < 2 * R; ++i) {
    for (const void* q : {static_cast<const void*>(recv[i]), static_cast<const void*>(cursor[i])}) {
      cudaPointerAttributes a{};
      CK(cudaPointerGetAttributes(&a, q));
      if (a.type != cudaMemoryTypeDevice)
        return fail(LT_ERR_INVALID, "peer buffers and cursors must be device memory");
      if (a.device == ctx->cfg.device) continue;
      int can = 0;
      CK(cudaDeviceCanAccessPeer(&can, ctx->cfg.device, a.device));
      if (!can)
        return fail(LT_ERR_INVALID, "device " + std::to_string(ctx->cfg.device) + " cannot access peer device " +
                                        std::to_string(a.device));
      const cudaError_t e = cudaDeviceEnablePeerAccess(a.device, 0);
      if (e == cudaErrorPeerAccessAlreadyEnabled) (void)cudaGetLastError();
      else CK(e);
    }
  }
  if (!ctx->d_peer_recv) CK(cudaMalloc(&ctx->d_peer_recv, 2 * R * sizeof(uint4*)));
  if (!ctx->d_peer_cur) CK(cudaMalloc(&ctx->d_peer_cur, 2 * R * sizeof(unsigned long long*)));
  CK(cudaMemcpy(ctx->d_peer_recv, recv, 2 * R * sizeof(void*), cudaMemcpyHostToDevice));
  CK(cudaMemcpy(ctx->d_peer_cur, cursor, 2 * R * sizeof(void*), cudaMemcpyHostToDevice));
  ctx->peer_on = true;
  ctx->params.peer = lt::Peer{ctx->d_peer_recv, ctx->d_peer_cur, ctx->xcap, ctx->peer_epoch};
  return LT_OK;
}

lt_status lt_exchange_sent(lt_ctx* ctx, uint64_t* sent) {
  if (!ctx || !sent) return fail(LT_ERR_INVALID, "NULL argument");
  if (!ctx->walks_ready) return fail(LT_ERR_STATE, "no walks");
  CK(cudaSetDevice(ctx->cfg.device));
  lt_status st = lt::snapshot_cached(ctx);
  if (st != LT_OK) return st;
  if (ctx->h_ctr->err & lt::kErrPeer) return fail(LT_ERR_INVALID, "a peer receive buffer overflowed; raise its capacity");
  *sent = ctx->h_ctr->sent;
  return LT_OK;
}

lt_status lt_exchange_take(lt_ctx* ctx, uint64_t* received) {
  if (!ctx || !received) return fail(LT_ERR_INVALID, "NULL argument");
  if (!ctx->peer_on) return fail(LT_ERR_STATE, "lt_exchange_take before lt_exchange_attach");
  if (!ctx->walks_ready) return fail(LT_ERR_STATE, "no walks");
  CK(cudaSetDevice(ctx->cfg.device));
  const uint32_t e = ctx->peer_epoch;
  unsigned long long cnt = 0;
  CK(cudaMemcpyAsync(&cnt, ctx->d_xcur + e * kXcurStride, sizeof(cnt), cudaMemcpyDeviceToHost, ctx->stream));
  CK(cudaStreamSynchronize(ctx->stream));
  if (cnt > ctx->xcap) return fail(LT_ERR_INVALID, "a peer receive buffer overflowed; raise its capacity");
  if (cnt) {
    ctx->snap_valid = false;
    CK(lt::launch_insert_records(ctx->params, ctx->d_xbuf[e], cnt, ctx->stream));
    ctx->stats.kernel_launches++;
  }
  // stream-ordered after the insert: the buffer of epoch e is written again only in superstep s + 2,
  // whose senders start after this rank's next lt_run (hence this reset) has completed
  CK(cudaMemsetAsync(ctx->d_xcur + e * kXcurStride, 0, sizeof(unsigned long long), ctx->stream));
  CK(cudaMemsetAsync(&ctx->d_ctr->sent, 0, sizeof(unsigned long long), ctx->stream));
  ctx->snap_valid = false;
  ctx->peer_epoch ^= 1u;
  ctx->params.peer.epoch = ctx->peer_epoch;
  *received = cnt;
  return LT_OK;
}

lt_status lt_superstep_p2p(lt_ctx* ctx, unsigned long long* d_sent) {
  if (!ctx || !d_sent) return fail(LT_ERR_INVALID, "NULL argument");
  if (!ctx->peer_on) return fail(LT_ERR_STATE, "lt_superstep_p2p before lt_exchange_attach");
  if (!ctx->walks_ready) return fail(LT_ERR_STATE, "no walks");
  if (ctx->own_hi - ctx->own_lo != 1 || ctx->ooc.on || ctx->cap_walks < ctx->W)
    return fail(LT_ERR_INVALID, "lt_superstep_p2p needs one owned partition per rank, an HBM-resident graph "
                                "and no walk-pool cap; use lt_run + lt_exchange_take");
  CK(cudaSetDevice(ctx->cfg.device));
  cudaStream_t s = ctx->stream;
  // (1) the walks peers appended in the previous superstep (parity epoch ^ 1) into the owned bucket
  const uint32_t prev = ctx->peer_epoch ^ 1u;
  CK(lt::launch_insert_records_dev(ctx->params, ctx->d_xbuf[prev], ctx->d_xcur + prev * kXcurStride, s));
  CK(cudaMemsetAsync(ctx->d_xcur + prev * kXcurStride, 0, sizeof(unsigned long long), s));
  CK(cudaMemsetAsync(&ctx->d_ctr->sent, 0, sizeof(unsigned long long), s));
  // (2) every owned walk steps until it ends or leaves for a peer (parity epoch), in one launch: the
  // owned bucket is the only one this rank consumes and walks stay in the kernel while inside it
  ctx->params.peer.epoch = ctx->peer_epoch;
  lt_status st = lt::launch_update_timed(ctx, ctx->params, ctx->own_lo, ~0ull >> 8);
  if (st != LT_OK) return st;
  CK(cudaMemcpyAsync(d_sent, &ctx->d_ctr->sent, sizeof(unsigned long long), cudaMemcpyDeviceToDevice, s));
  ctx->stats.kernel_launches += 1;
  ctx->snap_valid = false;
  ctx->peer_epoch ^= 1u;
  ctx->params.peer.epoch = ctx->peer_epoch;
  return LT_OK;
}

// ---- paths on the home rank (range ownership): every rank's path entries and lengths are written into
// one rank's matrix over peer memory, so no cross-rank merge is needed
lt_status lt_paths_buffers(lt_ctx* ctx, void** d_paths, void** d_lengths, uint64_t* capacity) {
  if (!ctx || !d_paths || !d_lengths || !capacity) return fail(LT_ERR_INVALID, "NULL argument");
  if (!ctx->walks_ready) return fail(LT_ERR_STATE, "lt_paths_buffers before lt_walks_init");
  if (ctx->cfg.path_mode == 2) return fail(LT_ERR_STATE, "paths are not stored (path_mode 2)");
  if (ctx->home_paths) return fail(LT_ERR_STATE, "this rank writes into another rank's matrix");
  if (ctx->arena)
    return fail(LT_ERR_STATE, "with a caller arena the path matrix is a sub-allocation: CUDA IPC needs its own");
  ctx->is_home = true;
  *d_paths = ctx->d_paths;
  *d_lengths = ctx->d_lengths;
  *capacity = ctx->paths_cap;
  return LT_OK;
}

lt_status lt_paths_attach(lt_ctx* ctx, void* d_paths, void* d_lengths, uint64_t capacity) {
  if (!ctx) return fail(LT_ERR_INVALID, "NULL ctx");
  if ((d_paths == nullptr) != (d_lengths == nullptr)) return fail(LT_ERR_INVALID, "pass both buffers or neither");
  if (d_paths && ctx->world < 2) return fail(LT_ERR_INVALID, "lt_paths_attach needs world > 1");
  if (d_paths && ctx->cfg.path_mode == 2) return fail(LT_ERR_STATE, "paths are not stored (path_mode 2)");
  if (d_paths && ctx->walks_ready && ctx->cfg.path_mode == 1)
    return fail(LT_ERR_STATE, "path_mode 1 writes path[w][0] in lt_walks_init: attach before it");
  CK(cudaSetDevice(ctx->cfg.device));
  if (d_paths) {
    for (const void* q : {static_cast<const void*>(d_paths), static_cast<const void*>(d_lengths)}) {
      cudaPointerAttributes a{};
      CK(cudaPointerGetAttributes(&a, q));
      if (a.type != cudaMemoryTypeDevice) return fail(LT_ERR_INVALID, "home buffers must be device memory");
      if (a.device != ctx->cfg.device) {
        int can = 0;
        CK(cudaDeviceCanAccessPeer(&can, ctx->cfg.device, a.device));
        if (!can) return fail(LT_ERR_INVALID, "no peer access to the home rank's device");
        const cudaError_t e = cudaDeviceEnablePeerAccess(a.device, 0);
        if (e == cudaErrorPeerAccessAlreadyEnabled) (void)cudaGetLastError();
        else CK(e);
      }
    }
  }
  ctx->home_paths = (uint32_t*)d_paths;
  ctx->home_lengths = (uint32_t*)d_lengths;
  ctx->home_cap = d_paths ? capacity : 0;
  if (ctx->walks_ready) {  // the current epoch writes there from the next launch on
    const bool home = d_paths != nullptr;
    if (home && ctx->W * (uint64_t)ctx->pitch > capacity)
      return fail(LT_ERR_INVALID, "the home rank's path matrix is smaller than W x pitch");
    ctx->params.wk.paths = home ? ctx->home_paths : ctx->d_paths;
    ctx->params.wk.lengths = home ? ctx->home_lengths : ctx->d_lengths;
    ctx->params.sys_fence = home ? 1u : 0u;
  }
  return LT_OK;
}

lt_status lt_ipc_handle(const void* dptr, void* handle) {
  if (!dptr || !handle) return fail(LT_ERR_INVALID, "NULL argument");
  cudaIpcMemHandle_t h;
  CK(cudaIpcGetMemHandle(&h, const_cast<void*>(dptr)));
  std::memcpy(handle, &h, sizeof(h));
  return LT_OK;
}

lt_status lt_ipc_open(lt_ctx* ctx, const void* handle, void** dptr) {
  if (!ctx || !handle || !dptr) return fail(LT_ERR_INVALID, "NULL argument");
  CK(cudaSetDevice(ctx->cfg.device));
  cudaIpcMemHandle_t h;
  std::memcpy(&h, handle, sizeof(h));
  void* q = nullptr;
  CK(cudaIpcOpenMemHandle(&q, h, cudaIpcMemLazyEnablePeerAccess));
  ctx->ipc_opened.push_back(q);
  *dptr = q;
  return LT_OK;
}

// lt_run_to_host / lt_run_to_host_compact: dense rows (paths != NULL) or the ragged layout
// (offsets != NULL: offsets[W+1] + vertices[<= vcap]).
static lt_status run_to_host_impl(lt_ctx* ctx, uint64_t W, const uint32_t* starts, uint64_t first_walk_id, lt_app app,
                                  double param, uint64_t seed, uint32_t* paths, uint32_t* lengths, uint64_t* offsets,
                                  uint32_t* vertices, uint64_t vcap, uint32_t chunks) {
  if (!ctx) return fail(LT_ERR_INVALID, "NULL ctx");
  if (ctx->world != 1) return fail(LT_ERR_INVALID, "lt_run_to_host needs a single-rank context");
  const bool compact = offsets != nullptr;
  if (W && (!starts || (!compact && (!paths || !lengths)))) return fail(LT_ERR_INVALID, "NULL argument");
  if (compact && vcap && !vertices) return fail(LT_ERR_INVALID, "NULL vertices");
  if (!ctx->graph_loaded) return fail(LT_ERR_STATE, "lt_run_to_host before lt_graph_load");
  if (ctx->cfg.visit_counts) return fail(LT_ERR_INVALID, "lt_run_to_host does not accumulate visit counts; use lt_run");
  if (ctx->cfg.path_mode == 2) return fail(LT_ERR_INVALID, "lt_run_to_host needs stored paths (path_mode 0 or 1)");
  if (app != LT_APP_DEEPWALK && app != LT_APP_PPR)
    return fail(LT_ERR_INVALID, "lt_run_to_host runs DeepWalk or PPR walks (PageRank: lt_walks_init_pagerank + lt_run)");
  CK(cudaSetDevice(ctx->cfg.device));
  if (chunks == 0) chunks = 8;
  const uint64_t wc = std::max<uint64_t>((W + chunks - 1) / chunks, 1);
  if (!ctx->copy_stream) {
    CK(cudaStreamCreateWithFlags(&ctx->copy_stream, cudaStreamNonBlocking));
    for (int i = 0; i < 2; ++i) {
      CK(cudaEventCreateWithFlags(&ctx->ev_computed[i], cudaEventDisableTiming));
      CK(cudaEventCreateWithFlags(&ctx->ev_copied[i], cudaEventDisableTiming));
      CK(cudaEventRecord(ctx->ev_copied[i], ctx->copy_stream));
    }
  }
  // All starts go H2D once (pinned host memory: at the link rate) and are range-checked on the device,
  // instead of a host loop over W starts in front of every range's walk: each range then starts from
  // its slice of the validated device array.
  CK(ensure(ctx, ctx->d_starts_all, ctx->starts_all_cap, std::max<uint64_t>(W, 1)));
  if (W) {
    CK(cudaMemcpyAsync(ctx->d_starts_all, starts, W * sizeof(uint32_t), cudaMemcpyHostToDevice, ctx->stream));
    CK(cudaMemsetAsync(ctx->d_small + 2, 0, sizeof(uint32_t), ctx->stream));
    CK(lt::launch_check_starts(ctx->d_starts_all, W, ctx->n, ctx->d_small + 2, ctx->stream));
    uint32_t bad = 0;
    CK(cudaMemcpyAsync(&bad, ctx->d_small + 2, sizeof(uint32_t), cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
    if (bad) return fail(LT_ERR_INVALID, "a start vertex >= n");
  }
  // the chunk buffers stand in for the context's path/length arrays while this call runs
  uint32_t* save_p = ctx->d_paths;
  size_t save_pc = ctx->paths_cap;
  uint32_t* save_l = ctx->d_lengths;
  size_t save_lc = ctx->lengths_cap;
  uint64_t steps = 0, visits = 0, trunc = 0, launches = 0, upd = 0, sweeps = 0, h2d = 0, d2h = 0;
  double run_ms = 0, init_ms = 0, update_ms = 0;
  lt_status st = LT_OK;
  uint64_t vbase = 0;  // compact: vertices written before this range
  for (uint64_t a = 0, c = 0; a < W || (W == 0 && c == 0); a += wc, ++c) {
    const uint64_t n = std::min<uint64_t>(wc, W - a);
    const int b = (int)(c & 1);
    CK(cudaEventSynchronize(ctx->ev_copied[b]));  // buffer b's previous chunk reached the host
    ctx->d_paths = ctx->d_paths2[b];
    ctx->paths_cap = ctx->paths2_cap[b];
    ctx->d_lengths = ctx->d_lengths2[b];
    ctx->lengths_cap = ctx->lengths2_cap[b];
    st = app == LT_APP_DEEPWALK
             ? walks_init_impl(ctx, n, ctx->d_starts_all + a, 2, first_walk_id + a, app, param, 0.0, seed)
             : walks_init_impl(ctx, n, ctx->d_starts_all + a, 2, first_walk_id + a, app, 0.0, param, seed);
    if (st == LT_OK) st = lt_run(ctx);
    ctx->d_paths2[b] = ctx->d_paths;  // (re)allocated by walks_init as needed
    ctx->paths2_cap[b] = ctx->paths_cap;
    ctx->d_lengths2[b] = ctx->d_lengths;
    ctx->lengths2_cap[b] = ctx->lengths_cap;
    if (st != LT_OK) break;
    steps += ctx->stats.steps;
    visits += ctx->stats.visits;
    trunc += ctx->stats.truncated;
    launches += ctx->stats.kernel_launches;
    upd += ctx->stats.update_launches;
    sweeps += ctx->stats.sweeps;
    run_ms += ctx->stats.run_ms;
    init_ms += ctx->stats.init_ms;
    update_ms += ctx->stats.update_ms;

    if (n && compact) {  // ragged copy-out: offsets + packed vertices of this range
      uint64_t tot = 0;
      st = pack_compact(ctx, ctx->d_paths2[b], ctx->d_lengths2[b], n, b, vbase, &tot);
      if (st != LT_OK) break;
      if (vbase + tot > vcap) {
        st = fail(LT_ERR_INVALID, "vertices buffer too small");
        break;
      }
      CK(cudaEventRecord(ctx->ev_computed[b], ctx->stream));
      CK(cudaStreamWaitEvent(ctx->copy_stream, ctx->ev_computed[b], 0));
      CK(cudaMemcpyAsync(offsets + a, ctx->d_off2[b], n * sizeof(uint64_t), cudaMemcpyDeviceToHost, ctx->copy_stream));
      if (tot)
        CK(cudaMemcpyAsync(vertices + vbase, ctx->d_vert2[b], tot * sizeof(uint32_t), cudaMemcpyDeviceToHost,
                           ctx->copy_stream));
      CK(cudaEventRecord(ctx->ev_copied[b], ctx->copy_stream));
      vbase += tot;
      d2h += n * 8 + tot * 4;
    } else if (n) {  // stream chunk c out while chunk c+1 computes
      // dense rows first (a 2-D copy of 324-B rows runs well below the link rate)
      CK(ensure(ctx, ctx->d_dense2[b], ctx->dense2_cap[b], n * ctx->stride));
      CK(lt::launch_compact_rows(ctx->d_paths2[b], ctx->d_lengths2[b], ctx->pitch, ctx->stride, n, ctx->d_dense2[b],
                                 ctx->stream));
      CK(cudaEventRecord(ctx->ev_computed[b], ctx->stream));
      CK(cudaStreamWaitEvent(ctx->copy_stream, ctx->ev_computed[b], 0));
      CK(cudaMemcpyAsync(paths + a * ctx->stride, ctx->d_dense2[b], n * ctx->stride * sizeof(uint32_t),
                         cudaMemcpyDeviceToHost, ctx->copy_stream));
      CK(cudaMemcpyAsync(lengths + a, ctx->d_lengths2[b], n * sizeof(uint32_t), cudaMemcpyDeviceToHost,
                         ctx->copy_stream));
      CK(cudaEventRecord(ctx->ev_copied[b], ctx->copy_stream));
      d2h += n * (ctx->stride + 1) * 4;
    }
    if (W == 0) break;
  }
  CK(cudaStreamSynchronize(ctx->copy_stream));
  if (compact && st == LT_OK) offsets[W] = vbase;
  ctx->d_paths = save_p;
  ctx->paths_cap = save_pc;
  ctx->d_lengths = save_l;
  ctx->lengths_cap = save_lc;
  ctx->walks_ready = false;  // the context's own path arrays do not hold these walks
  ctx->ran = false;
  if (st != LT_OK) return st;
  ctx->stats.num_walks = W;
  ctx->stats.steps = steps;
  ctx->stats.visits = visits;
  ctx->stats.truncated = trunc;
  ctx->stats.kernel_launches = launches;
  ctx->stats.update_launches = upd;
  ctx->stats.sweeps = sweeps;
  ctx->stats.run_ms = run_ms;
  ctx->stats.init_ms = init_ms;
  ctx->stats.update_ms = update_ms;
  ctx->stats.h2d_bytes = h2d + W * sizeof(uint32_t);
  ctx->stats.d2h_bytes = d2h;
  return LT_OK;
}

lt_status lt_run_to_host(lt_ctx* ctx, uint64_t W, const uint32_t* starts, uint64_t first_walk_id, lt_app app,
                         double param, uint64_t seed, uint32_t* paths, uint32_t* lengths, uint32_t chunks) {
  return run_to_host_impl(ctx, W, starts, first_walk_id, app, param, seed, paths, lengths, nullptr, nullptr, 0, chunks);
}

lt_status lt_run_to_host_compact(lt_ctx* ctx, uint64_t W, const uint32_t* starts, uint64_t first_walk_id, lt_app app,
                                 double param, uint64_t seed, uint64_t* offsets, uint32_t* vertices,
                                 uint64_t vertices_capacity, uint32_t chunks) {
  if (!offsets) return fail(LT_ERR_INVALID, "NULL offsets");
  return run_to_host_impl(ctx, W, starts, first_walk_id, app, param, seed, nullptr, nullptr, offsets, vertices,
                          vertices_capacity, chunks);
}

static lt_status copy_visits(lt_ctx* ctx, uint64_t* counts, cudaMemcpyKind kind) {
  if (!ctx || !counts) return fail(LT_ERR_INVALID, "NULL argument");
  if (!ctx->cfg.visit_counts) return fail(LT_ERR_STATE, "visit counting is off (lt_config.visit_counts)");
  if (!ctx->visits_ready) return fail(LT_ERR_STATE, "visit counts requested before lt_run");
  CK(cudaSetDevice(ctx->cfg.device));
  CK(cudaMemcpyAsync(counts, ctx->d_visits, (size_t)ctx->n * sizeof(uint64_t), kind, ctx->stream));
  if (kind == cudaMemcpyDeviceToHost) ctx->stats.d2h_bytes += (uint64_t)ctx->n * 8;
  CK(cudaStreamSynchronize(ctx->stream));
  return LT_OK;
}

lt_status lt_get_visit_counts(lt_ctx* ctx, uint64_t* counts) { return copy_visits(ctx, counts, cudaMemcpyDeviceToHost); }

lt_status lt_get_visit_counts_device(lt_ctx* ctx, uint64_t* d_counts) {
  return copy_visits(ctx, d_counts, cudaMemcpyDeviceToDevice);
}

lt_status lt_philox_device(int device, uint64_t n, const uint32_t* ctr, const uint32_t* key, uint32_t* out) {
  if (n && (!ctr || !key || !out)) return fail(LT_ERR_INVALID, "NULL argument");
  if (!n) return LT_OK;
  CK(cudaSetDevice(device));
  uint4* d_ctr = nullptr;
  uint2* d_key = nullptr;
  uint4* d_out = nullptr;
  cudaError_t e = cudaMalloc((void**)&d_ctr, n * sizeof(uint4));
  if (e == cudaSuccess) e = cudaMalloc((void**)&d_key, n * sizeof(uint2));
  if (e == cudaSuccess) e = cudaMalloc((void**)&d_out, n * sizeof(uint4));
  if (e == cudaSuccess) e = cudaMemcpy(d_ctr, ctr, n * sizeof(uint4), cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = cudaMemcpy(d_key, key, n * sizeof(uint2), cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = lt::launch_philox_blocks(d_ctr, d_key, d_out, n, nullptr);
  if (e == cudaSuccess) e = cudaMemcpy(out, d_out, n * sizeof(uint4), cudaMemcpyDeviceToHost);
  cudaFree(d_ctr);
  cudaFree(d_key);
  cudaFree(d_out);
  if (e != cudaSuccess) return fail(LT_ERR_CUDA, std::string("lt_philox_device: ") + cudaGetErrorString(e));
  return LT_OK;
}

lt_status lt_get_stats(lt_ctx* ctx, lt_stats* out) {
  if (!ctx || !out) return fail(LT_ERR_INVALID, "NULL argument");
  ctx->stats.arena_bytes_used = ctx->arena ? ctx->arena_peak : 0;
  *out = ctx->stats;
  return LT_OK;
}

}  // extern "C"

// The compressed-partition encoder on one column slice (host only; tests and tools): *words receives the
// payload length; hdr must hold ceil(len / 32) + 1 entries (2 u32 each: first value, payload word offset),
// pay (may be NULL to query *words) at least *words u32.
lt_status lt_compress_columns(const uint32_t* col, uint64_t len, uint32_t* hdr, uint32_t* pay, uint64_t* words) {
  if ((len && !col) || !words) return fail(LT_ERR_INVALID, "NULL argument");
  const uint64_t nblk = (len + 31) / 32;
  std::vector<uint8_t> w(nblk);
  uint64_t tot = 0;
  for (uint64_t j = 0; j < nblk; ++j) {
    w[j] = (uint8_t)block_width(col + 32 * j, std::min<uint64_t>(32, len - 32 * j));
    tot += w[j];
  }
  *words = tot;
  if (!pay) return LT_OK;
  if (!hdr) return fail(LT_ERR_INVALID, "NULL hdr");
  if (tot >= 0xFFFFFFFFull) return fail(LT_ERR_INVALID, "slice too large for 32-bit payload offsets");
  encode_slice(col, len, w.data(), reinterpret_cast<uint2*>(hdr), pay);
  return LT_OK;
}
