// lt_sched.cpp — the host partition scheduler (Alg. 2).
//
// Resident mode (the graph is in HBM): sweeps over the partitions with pending walks, in descending
// pending order (selective) or ID order (round robin, :341), one update launch each.
//
// Out-of-core mode (cfg.graph_pool_bytes > 0): the CSR lives in pinned host memory (G_cpu, :112,
// :214); a graph pool of m_g blocks caches partitions on the device (:112-118). Each iteration
// picks a partition (selective: the most pending walks; round robin otherwise), makes it resident
// by an explicit cudaMemcpyAsync on the load stream into a free block or the block of the resident
// partition with the fewest pending walks (selective) / the oldest one (FIFO) (:200), or reads it
// through zero copy when alpha * w < S_p (adaptive scheduling, :263-265); while the load is in
// flight it runs ready resident partitions (preemptive scheduling, :194-198, Alg. 2 l.7-10).
// Cross-stream dependencies use events: a block is overwritten only after its last compute use,
// and a partition is computed only after its load finished (:208).
#include "lt_ctx.h"

#include <nvtx3/nvToolsExt.h>

#include <cstring>

namespace lt {

namespace {

lt_status read_counts(lt_ctx* ctx) {
  lt_status st = snapshot(ctx);
  if (st != LT_OK) return st;
  ctx->stats.chunks_free_min = std::min<uint64_t>(ctx->stats.chunks_free_min, (uint64_t)std::max(*ctx->h_free, 0));
  return LT_OK;
}

inline uint64_t pending(const lt_ctx* ctx, uint32_t k) { return ctx->h_hc[ctx->nb + k] - ctx->h_hc[k]; }

// cudaEventQuery without leaving cudaErrorNotReady behind for the next launch check
bool event_done(cudaEvent_t e) {
  const cudaError_t r = cudaEventQuery(e);
  if (r == cudaErrorNotReady) (void)cudaGetLastError();
  return r == cudaSuccess;
}

}  // namespace

Range::Range(const char* name) { nvtxRangePushA(name); }
Range::~Range() { nvtxRangePop(); }

lt_status snapshot(lt_ctx* ctx) {
  Range r("lt snapshot (host round trip)");
  ctx->stats.host_syncs++;
  unsigned long long* dh = nullptr;
  Counters* dc = nullptr;
  int* df = nullptr;
  CK(cudaHostGetDevicePointer((void**)&dh, ctx->h_hc, 0));
  CK(cudaHostGetDevicePointer((void**)&dc, ctx->h_ctr, 0));
  CK(cudaHostGetDevicePointer((void**)&df, ctx->h_free, 0));
  CK(launch_snapshot(ctx->d_hc, ctx->nb, ctx->hs, ctx->d_ctr, (const int*)ctx->d_small, dh, dc, df, ctx->stream));
  ctx->stats.kernel_launches++;
  CK(cudaStreamSynchronize(ctx->stream));
  ctx->snap_valid = true;
  return LT_OK;
}

// Every launch that moves walks between buckets (update, init, insert, pack) clears snap_valid; the
// ABI calls that only need the counts (lt_pending, lt_exchange_pack, the end of lt_run) then reuse the
// mirror instead of another D2H + stream synchronisation.
lt_status snapshot_cached(lt_ctx* ctx) { return ctx->snap_valid ? LT_OK : snapshot(ctx); }

// Walk admission (f3; lt_config.walk_pool_walks): create the next walks in index order once at least a
// quarter of the pool (or everything still to come) has room, so live walks never exceed cap_walks.
lt_status admit_walks(lt_ctx* ctx, uint64_t live, bool* did) {
  *did = false;
  ctx->stats.peak_live = std::max<uint64_t>(ctx->stats.peak_live, live);
  if (ctx->admitted >= ctx->W || live >= ctx->cap_walks) return LT_OK;
  const uint64_t room = ctx->cap_walks - live, rest = ctx->W - ctx->admitted;
  if (room < std::min<uint64_t>(rest, std::max<uint64_t>(ctx->cap_walks / 4, 1))) return LT_OK;
  const uint64_t n = std::min(room, rest);
  ctx->snap_valid = false;
  CK(launch_init(ctx->params, ctx->adm_starts + ctx->admitted, n, ctx->admitted, ctx->stream));
  ctx->admitted += n;
  ctx->stats.admissions++;
  ctx->stats.kernel_launches++;
  *did = true;
  return LT_OK;
}

// ------------------------------------------------------------------------------- walk spill (f3)
// The walk pool evicts whole chunks to pinned host memory when it is full and loads a partition's
// evicted chunks back before that partition is computed (reading R17:
// the chunks of the buckets with the fewest pending walks go first). Chunk c of bucket q may be evicted
// only when it lies wholly inside [head_q, cursor_q) — full and never written again (appends go to the
// cursor's chunk or later) — and q is not being launched; its ring slot then holds kSpilled and its
// device chunk is free. A launch of partition k consumes [head_k, tail_cap): every chunk there is on the
// device (tail_cap = the start of k's first chunk still on the host, or the prefix the free chunks can
// absorb). Eviction: k_spill copies the chunks into their host slots through the host store's device
// mapping and frees them (ring slot -> kSpilled); reload: k_reload copies host slots into fresh device
// chunks and installs them. Both run on the compute stream, so host slots and device chunks are reused in
// stream order, with no staging buffers and no per-chunk cudaMemcpy calls.
namespace {

// chunks a launch over n walks may need for its appends: one per C walks plus a partial tail chunk
// per destination bucket
inline uint64_t append_chunks(const lt_ctx* ctx, uint64_t n) {
  const uint64_t C = ctx->params.pool.C;
  return (n + C - 1) / C + ctx->nb + 1;
}

// Evict up to `want` chunks of buckets other than `keep` (fewest pending walks first, highest chunk
// index first), or, with only >= 0, of bucket `only` from chunk index min_ci up. Uses the last snapshot's
// head/cursor. Returns the number evicted in *done.
lt_status evict_chunks(lt_ctx* ctx, int keep, uint64_t want, uint64_t* done, int only = -1, uint64_t min_ci = 0) {
  Range rg("lt walk spill: evict");
  Spill& sp = ctx->spill;
  const uint64_t C = ctx->params.pool.C;
  const uint32_t nb = ctx->nb;
  *done = 0;
  if (!want) return LT_OK;
  std::vector<uint32_t> order;
  for (uint32_t q = 0; q < nb; ++q)
    if ((int)q != keep && (only < 0 || (int)q == only) && ctx->h_hc[nb + q] > ctx->h_hc[q]) order.push_back(q);
  // reading R17: out of core, the buckets of partitions whose graph is NOT in the graph pool go first (a
  // resident partition is likely computed soon); then the fewest pending walks
  auto resident = [&](uint32_t q) { return ctx->ooc.on && q < ctx->P && ctx->ooc.block_of[q] >= 0; };
  std::stable_sort(order.begin(), order.end(), [&](uint32_t a, uint32_t b) {
    if (resident(a) != resident(b)) return !resident(a);
    return ctx->h_hc[nb + a] - ctx->h_hc[a] < ctx->h_hc[nb + b] - ctx->h_hc[b];
  });
  SpillList list;
  uint32_t cnt = 0;
  auto flush = [&]() -> lt_status {
    if (!cnt) return LT_OK;
    const cudaStream_t s = ctx->stream;
    if (ctx->cfg.timing) CK(ctx->xfer_ev.begin(s));
    CK(launch_spill(ctx->params, list, cnt, sp.d_store, s));
    if (ctx->cfg.timing) CK(ctx->xfer_ev.end(s));
    sp.host_used += cnt;
    sp.free_chunks += cnt;
    ctx->stats.spilled_chunks += cnt;
    ctx->stats.spill_d2h_bytes += (uint64_t)cnt * C * sizeof(uint4);
    ctx->stats.host_chunks_peak = std::max<uint64_t>(ctx->stats.host_chunks_peak, sp.host_used);
    ctx->stats.kernel_launches++;
    ctx->snap_valid = false;
    cnt = 0;
    return LT_OK;
  };
  for (uint32_t q : order) {
    const uint64_t head = ctx->h_hc[q], cur = ctx->h_hc[nb + q];
    const uint64_t lo = std::max<uint64_t>((head + C - 1) / C, min_ci);  // first chunk wholly at or after head
    const uint64_t hi = cur / C;             // chunks [lo, hi) end at or before cursor
    for (uint64_t ci = hi; ci-- > lo && *done < want;) {
      if (sp.spilled[q].count(ci)) continue;
      if (sp.host_free.empty()) return fail(LT_ERR_OOM, "walk spill: host store full (invariant violated)");
      const uint32_t hs = sp.host_free.back();  // host slots are reused in stream order (kernels only)
      sp.host_free.pop_back();
      sp.spilled[q][ci] = hs;
      list.bucket[cnt] = q;
      list.chunk[cnt] = ci;
      list.slot[cnt] = hs;
      ++*done;
      if (++cnt == kSpillBatch) {
        lt_status st = flush();
        if (st != LT_OK) return st;
      }
    }
    if (*done >= want) break;
  }
  return flush();
}

// Load the first r evicted chunks of bucket k (lowest chunk index first) back into device chunks.
lt_status reload_chunks(lt_ctx* ctx, uint32_t k, uint64_t r) {
  Range rg("lt walk spill: reload");
  Spill& sp = ctx->spill;
  const uint64_t C = ctx->params.pool.C;
  auto& sk = sp.spilled[k];
  while (r && !sk.empty()) {
    SpillList list;
    uint32_t cnt = 0;
    for (auto it = sk.begin(); it != sk.end() && cnt < kSpillBatch && cnt < r;) {
      list.bucket[cnt] = k;
      list.chunk[cnt] = it->first;
      list.slot[cnt] = it->second;
      sp.host_free.push_back(it->second);  // an eviction into this slot is stream-ordered after this reload
      it = sk.erase(it);
      ++cnt;
    }
    const cudaStream_t s = ctx->stream;
    if (ctx->cfg.timing) CK(ctx->xfer_ev.begin(s));
    CK(launch_reload(ctx->params, list, cnt, sp.d_store, s));
    if (ctx->cfg.timing) CK(ctx->xfer_ev.end(s));
    sp.host_used -= cnt;
    sp.free_chunks -= cnt;
    ctx->stats.reloaded_chunks += cnt;
    ctx->stats.spill_h2d_bytes += (uint64_t)cnt * C * sizeof(uint4);
    ctx->stats.kernel_launches++;
    ctx->snap_valid = false;
    r -= cnt;
  }
  return LT_OK;
}

// Before a launch of partition k: make [head_k, tail_cap) device-resident and leave enough free chunks
// for the launch's appends, evicting other buckets' chunks as needed. *tail_cap = ~0 when all of k fits.
lt_status ensure_walks(lt_ctx* ctx, uint32_t k, unsigned long long* tail_cap) {
  Spill& sp = ctx->spill;
  *tail_cap = ~0ull;
  lt_status st = snapshot(ctx);
  if (st != LT_OK) return st;
  sp.free_chunks = std::max(*ctx->h_free, 0);
  const uint64_t C = ctx->params.pool.C;
  const uint64_t head = ctx->h_hc[k], cur = ctx->h_hc[ctx->nb + k];
  auto& sk = sp.spilled[k];
  // (1) room for k's evicted chunks and every append of its launch: other buckets' chunks go first
  const int64_t want_free = (int64_t)(sk.size() + append_chunks(ctx, cur - head));
  if (sp.free_chunks < want_free) {
    uint64_t done = 0;
    st = evict_chunks(ctx, (int)k, (uint64_t)(want_free - sp.free_chunks), &done);
    if (st != LT_OK) return st;
  }
  // (2) the launch must make progress: room for one chunk of appends, plus k's first evicted chunk when
  // it starts at head. If the pool is still that full (k itself holds most chunks), k's own top chunks
  // above its first full chunk are evicted.
  const bool head_spilled = !sk.empty() && sk.begin()->first * C <= head;
  const int64_t min_free = (head_spilled ? 1 : 0) + (int64_t)ctx->nb + 2;
  if (sp.free_chunks < min_free) {
    uint64_t done = 0;
    st = evict_chunks(ctx, -1, (uint64_t)(min_free - sp.free_chunks), &done, (int)k, (head + C - 1) / C + 1);
    if (st != LT_OK) return st;
  }
  // (3) reload k's evicted chunks, lowest first, while the free chunks still absorb the appends of every
  // walk up to the end of the reloaded chunk
  uint64_t r = 0;
  for (auto it = sk.begin(); it != sk.end(); ++it) {
    const uint64_t walks_to = (it->first + 1) * C - head;
    if (sp.free_chunks < (int64_t)(r + 1 + append_chunks(ctx, walks_to))) break;
    ++r;
  }
  st = reload_chunks(ctx, k, r);
  if (st != LT_OK) return st;
  // (4) the launch stops at k's first chunk still on the host, or earlier if the free chunks cannot
  // absorb the appends of every device-resident walk before it
  unsigned long long cap = sk.empty() ? ~0ull : sk.begin()->first * C;
  const int64_t room = sp.free_chunks - (int64_t)ctx->nb - 1;  // chunks left for full chunks of appends
  if (room < 1) return fail(LT_ERR_OOM, "walk spill: the walk pool cannot hold one chunk of appends; raise walk_pool_walks");
  const unsigned long long fit = head + (unsigned long long)room * C;
  if (fit < std::min<unsigned long long>(cap, cur)) cap = fit;
  if (cap <= head) return fail(LT_ERR_OOM, "walk spill: no walk of the selected partition fits the walk pool");
  *tail_cap = cap;
  return LT_OK;
}

}  // namespace

lt_status spill_admit_all(lt_ctx* ctx) {
  Spill& sp = ctx->spill;
  const uint64_t C = ctx->params.pool.C;
  const uint64_t batch = std::max<uint64_t>(C, ctx->cap_walks / 2);
  while (ctx->admitted < ctx->W) {
    lt_status st = snapshot(ctx);
    if (st != LT_OK) return st;
    sp.free_chunks = std::max(*ctx->h_free, 0);
    const uint64_t n0 = std::min<uint64_t>(batch, ctx->W - ctx->admitted);
    const int64_t need = (int64_t)append_chunks(ctx, n0);  // a k_init of n walks appends like a launch
    if (sp.free_chunks < need) {
      uint64_t done = 0;
      st = evict_chunks(ctx, -1, (uint64_t)(need - sp.free_chunks), &done);
      if (st != LT_OK) return st;
    }
    const int64_t room = sp.free_chunks - (int64_t)ctx->nb - 1;
    if (room < 1) return fail(LT_ERR_OOM, "walk spill: the walk pool cannot hold one chunk of new walks");
    const uint64_t n = std::min<uint64_t>(n0, (uint64_t)room * C);
    ctx->snap_valid = false;
    CK(launch_init(ctx->params, ctx->adm_starts + ctx->admitted, n, ctx->admitted, ctx->stream));
    ctx->admitted += n;
    ctx->stats.admissions++;
    ctx->stats.kernel_launches++;
  }
  return LT_OK;
}

void free_spill(lt_ctx* ctx) {
  Spill& sp = ctx->spill;
  if (sp.h_store) cudaFreeHost(sp.h_store);
  sp = Spill();
}

lt_status launch_update_timed(lt_ctx* ctx, const Params& p, uint32_t k, uint64_t walks_bound) {
  cudaStream_t s = ctx->stream;
  const uint64_t max_grid = (uint64_t)ctx->num_sms * ctx->occ;
  const uint64_t per_block = (uint64_t)ctx->block * p.ilp;
  const uint64_t grid = std::min<uint64_t>(std::max<uint64_t>((walks_bound + per_block - 1) / per_block, 1), max_grid);
  if (ctx->cfg.timing) {
    while (ctx->events.size() < ctx->nev + 2) {
      cudaEvent_t ev;
      CK(cudaEventCreate(&ev));
      ctx->events.push_back(ev);
    }
    CK(cudaEventRecord(ctx->events[ctx->nev], s));
  }
  ctx->snap_valid = false;
  Range rg("lt update launch");
  CK(launch_update(p, k, (uint32_t)grid, ctx->block, s));
  if (ctx->cfg.timing) {
    CK(cudaEventRecord(ctx->events[ctx->nev + 1], s));
    ctx->nev += 2;
  }
  ctx->stats.update_launches++;
  ctx->stats.kernel_launches++;
  return LT_OK;
}

// Walk-spill prefetch: while partition k's launch runs, load back the evicted chunks of the partition
// most likely to be computed next (the most pending walks, as the selective policy picks),
// so its reload H2D overlaps k's compute instead of sitting in front of its own launch. Only chunks the
// free pool can spare beyond k's appends (up to ⌈launched/C⌉ + nb + 1 chunks) are loaded; the reload
// kernel is stream-ordered after k's launch. Parity-neutral: only residency changes.
static lt_status prefetch_walks(lt_ctx* ctx, uint32_t k, uint64_t launched) {
  Spill& sp = ctx->spill;
  int j = -1;
  uint64_t best = 0;
  for (uint32_t q = ctx->own_lo; q < ctx->own_hi; ++q) {
    if (q == k || sp.spilled[q].empty()) continue;
    const uint64_t pend = ctx->h_hc[ctx->nb + q] - ctx->h_hc[q];
    if (pend > best) {
      best = pend;
      j = (int)q;
    }
  }
  if (j < 0) return LT_OK;
  const int64_t spare = sp.free_chunks - (int64_t)append_chunks(ctx, launched) - (int64_t)ctx->nb - 2;
  if (spare <= 0) return LT_OK;
  const uint64_t r = std::min<uint64_t>((uint64_t)spare, sp.spilled[(uint32_t)j].size());
  ctx->stats.spill_prefetched_chunks += r;
  return reload_chunks(ctx, (uint32_t)j, r);
}

// One partition's update launch; with walk spill, as many launches as it takes to consume every walk
// that was in bucket k when the call began (each preceded by ensure_walks).
lt_status launch_partition(lt_ctx* ctx, const Params& p, uint32_t k, uint64_t walks_bound) {
  if (!ctx->spill.on) return launch_update_timed(ctx, p, k, walks_bound);
  Params pv = p;
  unsigned long long end = 0;
  for (bool first = true;; first = false) {
    unsigned long long cap = ~0ull;
    lt_status st = ensure_walks(ctx, k, &cap);
    if (st != LT_OK) return st;
    const unsigned long long head = ctx->h_hc[k], cur = ctx->h_hc[ctx->nb + k];
    if (first) end = cur;
    if (head >= end || head >= cur) return LT_OK;
    pv.tail_cap = cap;
    const unsigned long long launched = std::min<unsigned long long>(cap, cur) - head;
    st = launch_update_timed(ctx, pv, k, launched);
    if (st != LT_OK) return st;
    if (cap >= cur) return prefetch_walks(ctx, k, launched);
  }
}

lt_status run_resident(lt_ctx* ctx) {
  Range rg("lt run (HBM-resident scheduler)");
  const uint64_t max_len = (ctx->app == LT_APP_PPR) ? ctx->lmax : ctx->length;
  std::vector<uint32_t> order;
  order.reserve(ctx->P);
  uint64_t since_admission = 0;
  for (;;) {
    lt_status st = read_counts(ctx);  // one small D2H + sync per sweep
    if (st != LT_OK) return st;
    if (ctx->h_ctr->err) return LT_OK;
    order.clear();
    uint64_t total = 0;
    for (uint32_t k = ctx->own_lo; k < ctx->own_hi; ++k)  // owned partitions (all when world == 1)
      if (pending(ctx, k)) { order.push_back(k); total += pending(ctx, k); }
    bool admitted = false;
    st = admit_walks(ctx, total, &admitted);
    if (st != LT_OK) return st;
    if (admitted) {  // recount with the new walks in their buckets
      since_admission = 0;
      continue;
    }
    if (total == 0) return LT_OK;
    // every live walk advances >= 1 step per sweep, so sweeps <= max_len + 1 between admissions
    if (++since_admission > max_len + 3) return fail(LT_ERR_CUDA, "scheduler did not converge");
    if (ctx->cfg.policy == LT_POLICY_SELECTIVE || ctx->cfg.policy == LT_POLICY_SELECTIVE_ONLY)
      std::stable_sort(order.begin(), order.end(), [&](uint32_t a, uint32_t b) { return pending(ctx, a) > pending(ctx, b); });
    uint64_t earlier = 0;
    for (uint32_t k : order) {
      // walks present at launch time <= pending now + everything launched before in this sweep
      const uint64_t bound = pending(ctx, k) + earlier;
      earlier += pending(ctx, k);
      st = launch_partition(ctx, ctx->params, k, bound);
      if (st != LT_OK) return st;
    }
    ctx->stats.sweeps++;
  }
}

// ------------------------------------------------------------------------------- out-of-core
namespace {

uint64_t partition_bytes(const lt_ctx* ctx, uint32_t k) {
  const uint32_t v0 = ctx->h_bounds[k], v1 = ctx->h_bounds[k + 1];
  return 8ull * (v1 - v0 + 1) + 4ull * (ctx->ooc.h_row_ptr[v1] - ctx->ooc.h_row_ptr[v0]);
}

// bytes an explicit copy of partition k moves over the link (its compressed blocks when they are smaller)
uint64_t transfer_bytes(const lt_ctx* ctx, uint32_t k) {
  const OutOfCore& o = ctx->ooc;
  if (!o.comp || o.craw[k]) return partition_bytes(ctx, k);
  const uint32_t v0 = ctx->h_bounds[k], v1 = ctx->h_bounds[k + 1];
  return 8ull * (v1 - v0 + 1) + 8ull * (o.chdr_at[k + 1] - o.chdr_at[k]) + 4ull * (o.cpay_at[k + 1] - o.cpay_at[k]);
}

// Params whose graph view is partition k's slice in block b, or the whole mapped host CSR.
Params view_block(const lt_ctx* ctx, uint32_t k, int b) {
  Params p = ctx->params;
  const uint32_t v0 = ctx->h_bounds[k];
  char* base = ctx->ooc.d_gpool + (size_t)b * ctx->ooc.block_bytes;
  p.wk.row_ptr = reinterpret_cast<const unsigned long long*>(base);
  p.wk.col = reinterpret_cast<const uint32_t*>(base + ctx->ooc.rp_bytes);
  p.wk.vbase = v0;
  p.wk.ebase = ctx->ooc.h_row_ptr[v0];
  p.wk.adj = nullptr;
  return p;
}

Params view_zero_copy(const lt_ctx* ctx) {
  Params p = ctx->params;
  p.wk.row_ptr = ctx->ooc.d_map_row_ptr;
  p.wk.col = ctx->ooc.d_map_col;
  p.wk.vbase = 0;
  p.wk.ebase = 0;
  p.wk.adj = nullptr;
  return p;
}

// Continuation table (f4), kept on the compute stream: partition k's entry is published before a
// launch that may read its block — for the launched partition itself (the stream already waits for
// its load) and for every other resident partition whose load the host has seen complete — and
// withdrawn before its block is reloaded. Every launch may read any published block, so a reload
// waits for an event recorded on the compute stream after the withdrawal.
lt_status table_publish(lt_ctx* ctx, int launched) {
  OutOfCore& o = ctx->ooc;
  if (!ctx->params.cont.table) return LT_OK;
  uint32_t idx[kTableSetMax], val[kTableSetMax], cnt = 0;
  for (uint32_t q = 0; q < o.m_g; ++q) {
    const int k = o.part_in[q];
    if (k < 0 || o.table[k] == q) continue;
    if (k != launched && !event_done(o.ev_ready[q])) continue;
    o.table[k] = q;
    idx[cnt] = (uint32_t)k;
    val[cnt] = q;
    if (++cnt == kTableSetMax) {
      CK(launch_table_set(o.d_table, idx, val, cnt, ctx->stream));
      ctx->stats.kernel_launches++;
      cnt = 0;
    }
  }
  if (cnt) {
    CK(launch_table_set(o.d_table, idx, val, cnt, ctx->stream));
    ctx->stats.kernel_launches++;
  }
  return LT_OK;
}

lt_status load_partition(lt_ctx* ctx, uint32_t k, int b, uint64_t seq) {
  OutOfCore& o = ctx->ooc;
  const uint32_t v0 = ctx->h_bounds[k], v1 = ctx->h_bounds[k + 1];
  const uint64_t e0 = o.h_row_ptr[v0], e1 = o.h_row_ptr[v1];
  char* base = o.d_gpool + (size_t)b * o.block_bytes;
  const int old = o.part_in[b];
  if (ctx->params.cont.table && old >= 0 && o.table[old] != kEmpty) {  // withdraw the evicted partition
    const uint32_t idx = (uint32_t)old, val = kEmpty;
    CK(launch_table_set(o.d_table, &idx, &val, 1, ctx->stream));
    ctx->stats.kernel_launches++;
    o.table[old] = kEmpty;
    CK(cudaEventRecord(o.ev_used[b], ctx->stream));  // after every launch that could read the block
  }
  CK(cudaStreamWaitEvent(o.load_stream, o.ev_used[b], 0));  // the block's last reader is done
  Range rg("lt load partition (H2D)");
  if (ctx->cfg.timing) CK(ctx->load_ev.begin(o.load_stream));
  CK(cudaMemcpyAsync(base, o.h_row_ptr + v0, 8ull * (v1 - v0 + 1), cudaMemcpyHostToDevice, o.load_stream));
  if (e1 > e0 && o.comp && !o.craw[k]) {  // compressed blocks into the staging buffer, expanded into the block
    const uint64_t nh = o.chdr_at[k + 1] - o.chdr_at[k], nw = o.cpay_at[k + 1] - o.cpay_at[k];
    CK(cudaMemcpyAsync(o.d_cstage, o.h_chdr + o.chdr_at[k], nh * sizeof(uint2), cudaMemcpyHostToDevice, o.load_stream));
    if (nw)
      CK(cudaMemcpyAsync(o.d_cstage + nh * sizeof(uint2), o.h_cpay + o.cpay_at[k], nw * 4, cudaMemcpyHostToDevice,
                         o.load_stream));
    CK(launch_decode_cols(reinterpret_cast<const uint2*>(o.d_cstage),
                          reinterpret_cast<const uint32_t*>(o.d_cstage + nh * sizeof(uint2)), e1 - e0,
                          reinterpret_cast<uint32_t*>(base + o.rp_bytes), o.load_stream));
    ctx->stats.kernel_launches++;
  } else if (e1 > e0) {
    CK(cudaMemcpyAsync(base + o.rp_bytes, o.h_col + e0, 4ull * (e1 - e0), cudaMemcpyHostToDevice, o.load_stream));
  }
  if (ctx->cfg.timing) CK(ctx->load_ev.end(o.load_stream));
  CK(cudaEventRecord(o.ev_ready[b], o.load_stream));
  if (o.part_in[b] >= 0) o.block_of[o.part_in[b]] = -1;
  o.part_in[b] = (int)k;
  o.block_of[k] = b;
  o.loaded_at[b] = seq;
  ctx->stats.explicit_copies++;
  ctx->stats.graph_h2d_bytes += transfer_bytes(ctx, k);
  ctx->stats.graph_h2d_raw_bytes += partition_bytes(ctx, k);
  ctx->stats.h2d_bytes += transfer_bytes(ctx, k);
  return LT_OK;
}

lt_status compute_block(lt_ctx* ctx, uint32_t k) {
  OutOfCore& o = ctx->ooc;
  const int b = o.block_of[k];
  CK(cudaStreamWaitEvent(ctx->stream, o.ev_ready[b], 0));
  lt_status st = table_publish(ctx, (int)k);
  if (st != LT_OK) return st;
  st = launch_partition(ctx, view_block(ctx, k, b), k, pending(ctx, k));
  if (st != LT_OK) return st;
  CK(cudaEventRecord(o.ev_used[b], ctx->stream));
  return LT_OK;
}

// Prefetch (lt_config.ooc_prefetch): with partition i about to be computed and at most one load in
// flight (typically i's own), queue the load of the non-resident partition with the most pending walks (one a zero-copy launch would
// not serve) into a free block or the block of the resident partition with the fewest walks — never
// i's block. The victim is withdrawn from the continuation table BEFORE i's launch is enqueued, so the
// load only waits for the launches already issued and overlaps the compute of i. The next selection
// then usually finds that partition resident. Uses the counts of the last read (parity-neutral: only
// residency changes).
lt_status prefetch(lt_ctx* ctx, uint32_t i, bool selective, uint64_t alpha, uint64_t seq) {
  OutOfCore& o = ctx->ooc;
  if (!ctx->cfg.ooc_prefetch || o.m_g < 2) return LT_OK;
  uint32_t in_flight = 0;  // keep at most one load queued behind the one in flight
  for (uint32_t q = 0; q < o.m_g; ++q)
    if (o.part_in[q] >= 0 && !event_done(o.ev_ready[q])) ++in_flight;
  if (in_flight >= 2) return LT_OK;
  int j = -1;
  for (uint32_t k = ctx->own_lo; k < ctx->own_hi; ++k) {
    if (k == i || o.block_of[k] >= 0 || !pending(ctx, k)) continue;
    if (ctx->cfg.zero_copy && alpha * pending(ctx, k) < transfer_bytes(ctx, k)) continue;
    if (j < 0 || pending(ctx, k) > pending(ctx, (uint32_t)j)) j = (int)k;
  }
  if (j < 0) return LT_OK;
  const int bi = o.block_of[i];
  int b = -1;
  for (uint32_t q = 0; q < o.m_g && b < 0; ++q)
    if (o.part_in[q] < 0 && (int)q != bi) b = (int)q;
  if (b < 0) {
    for (uint32_t q = 0; q < o.m_g; ++q) {
      if ((int)q == bi) continue;
      if (b < 0) { b = (int)q; continue; }
      if (selective ? pending(ctx, o.part_in[q]) < pending(ctx, o.part_in[b]) : o.loaded_at[q] < o.loaded_at[b])
        b = (int)q;
    }
    // only displace a partition holding fewer walks than the one brought in
    if (b < 0 || pending(ctx, o.part_in[b]) >= pending(ctx, (uint32_t)j)) return LT_OK;
  }
  ctx->stats.prefetches++;
  lt_status st = load_partition(ctx, (uint32_t)j, b, seq);
  ctx->stats.explicit_copies--;  // explicit_copies counts the loads of selected partitions (Table III)
  return st;
}

}  // namespace

lt_status run_out_of_core(lt_ctx* ctx) {
  Range rg("lt run (out-of-core scheduler)");
  OutOfCore& o = ctx->ooc;
  const uint32_t P = ctx->P;
  const uint32_t pol = ctx->cfg.policy;
  const bool selective = pol == LT_POLICY_SELECTIVE || pol == LT_POLICY_SELECTIVE_ONLY;
  const bool preemptive = pol == LT_POLICY_SELECTIVE || pol == LT_POLICY_PREEMPTIVE_ONLY;
  const uint64_t alpha = ctx->cfg.zc_alpha_bytes ? ctx->cfg.zc_alpha_bytes : 256;
  const uint64_t max_len = (ctx->app == LT_APP_PPR) ? ctx->lmax : ctx->length;
  // each iteration consumes >= 1 visit and a walk makes <= max_len + 1 visits
  const uint64_t max_iters = ctx->W * (max_len + 1) + P + 64;
  uint64_t seq = 0;
  const uint32_t lo = ctx->own_lo, hi = ctx->own_hi;  // owned partitions (all when world == 1)
  uint32_t rr = hi - 1;  // round-robin cursor
  for (;;) {
    lt_status st = read_counts(ctx);  // Alg. 2 line 1: while active walks exist
    if (st != LT_OK) return st;
    if (ctx->h_ctr->err) return LT_OK;
    uint64_t total = 0;
    for (uint32_t k = lo; k < hi; ++k) total += pending(ctx, k);
    bool admitted = false;
    st = admit_walks(ctx, total, &admitted);
    if (st != LT_OK) return st;
    if (admitted) continue;
    if (total == 0) return LT_OK;
    if (ctx->stats.iterations > max_iters) return fail(LT_ERR_CUDA, "out-of-core scheduler did not converge");
    // scheduler.iteration(): select partition i
    uint32_t i = lo;
    if (selective) {
      for (uint32_t k = lo + 1; k < hi; ++k)
        if (pending(ctx, k) > pending(ctx, i)) i = k;
    } else {
      do { rr = (rr + 1 >= hi) ? lo : rr + 1; } while (!pending(ctx, rr));
      i = rr;
    }
    ctx->stats.iterations++;
    if (o.block_of[i] >= 0) {  // graph-pool hit
      ctx->stats.pool_hits++;
      st = prefetch(ctx, i, selective, alpha, ++seq);
      if (st != LT_OK) return st;
      st = compute_block(ctx, i);
      if (st != LT_OK) return st;
      continue;
    }
    // adaptive scheduling: zero copy when alpha * w < S_p (Alg. 2 l.3-4)
    if (ctx->cfg.zero_copy && alpha * pending(ctx, i) < transfer_bytes(ctx, i)) {
      ctx->stats.zero_copy_launches++;
      st = table_publish(ctx, -1);
      if (st != LT_OK) return st;
      st = launch_partition(ctx, view_zero_copy(ctx), i, pending(ctx, i));
      if (st != LT_OK) return st;
      continue;
    }
    // explicit copy (Alg. 2 l.6): a free block, else evict (fewest pending walks / FIFO)
    int b = -1;
    for (uint32_t q = 0; q < o.m_g && b < 0; ++q)
      if (o.part_in[q] < 0) b = (int)q;
    if (b < 0) {
      for (uint32_t q = 0; q < o.m_g; ++q) {
        if (b < 0) { b = (int)q; continue; }
        if (selective ? pending(ctx, o.part_in[q]) < pending(ctx, o.part_in[b]) : o.loaded_at[q] < o.loaded_at[b])
          b = (int)q;
      }
    }
    st = load_partition(ctx, i, b, ++seq);
    if (st != LT_OK) return st;
    // preemptive scheduling (Alg. 2 l.7-10): while the load stream is busy, run ready partitions
    while (preemptive && !event_done(o.ev_ready[b])) {
      int j = -1;
      // prefer a full batch whose partition holds the fewest walks, else the most walks
      const uint64_t full = ctx->params.pool.C;
      for (uint32_t q = 0; q < o.m_g; ++q) {
        const int k = o.part_in[q];
        if (k < 0 || (uint32_t)k == i || !pending(ctx, k)) continue;
        if (!event_done(o.ev_ready[q])) continue;
        if (j < 0) { j = k; continue; }
        const bool kf = pending(ctx, k) >= full, jf = pending(ctx, j) >= full;
        if (kf != jf ? kf : (kf ? pending(ctx, k) < pending(ctx, j) : pending(ctx, k) > pending(ctx, j))) j = k;
      }
      if (j < 0) break;
      ctx->stats.preemptive_launches++;
      st = compute_block(ctx, (uint32_t)j);
      if (st != LT_OK) return st;
      st = read_counts(ctx);  // Alg. 2 l.10: cudaStreamSynchronize(compStream)
      if (st != LT_OK) return st;
      if (ctx->h_ctr->err) return LT_OK;
    }
    st = prefetch(ctx, i, selective, alpha, ++seq);
    if (st != LT_OK) return st;
    st = compute_block(ctx, i);
    if (st != LT_OK) return st;
  }
}

}  // namespace lt
