/* lt.h — C ABI of the B200-native LightTraffic walk-update path (liblt.so).
 *
 * The path (BASELINE.json north_star): vertices of a CSR graph are split into
 * range partitions (§III-B "Graph data and partition"); walk states live in
 * per-partition buckets made of fixed-size chunks of a pool reserved up front (PAPER.md:118,
 * :124, :132-134, §III-B "Memory pool reservation" / "Walk index"); for each scheduled partition
 * a kernel advances every walk in that partition's bucket until it terminates or leaves the
 * partition (Alg. 1), and the updated walk is appended to the bucket
 * of its new partition (walk reshuffling, §III-C). The host scheduler picks
 * partitions by pending-walk count (selective scheduling) until no active walk
 * remains (Alg. 2 line 1).
 *
 * The walk itself (PAPER.md:45 §II-A; :287 §IV-A): uniform neighbour per step; DeepWalk stops after
 * l steps; PPR terminates with probability alpha before each move, capped at L_max steps. Sampling
 * is Philox4x32-10 keyed by (walk_id, step) plus Lemire's unbiased range reduction, so every path is
 * a pure function of (CSR, starts, app, parameter, seed, L_max) — independent of the partition
 * count, chunk size, scheduling policy and launch shape (readings R1-R6).
 *
 * Conventions for every function:
 *   - Returns lt_status; never aborts, never throws across the ABI. On error, lt_last_error()
 *     returns a thread-local message describing the first failure.
 *   - Host pointers are caller-owned and only read during the call (copied before return).
 *     "Device" pointers are CUDA device memory (e.g. torch tensors) that the caller keeps alive
 *     for as long as the context uses them; the library never frees them.
 *   - Call order: lt_create -> lt_graph_load* -> lt_walks_init* -> lt_run -> lt_get_* ;
 *     lt_walks_init* may be repeated after lt_run (a new epoch on the same graph). Out-of-order
 *     calls return LT_ERR_STATE. Device memory is reserved in lt_graph_load(_device) and lt_walks_init(_ex) only
 *     ("reserve the memory ... in advance"); lt_run never allocates.
 *   - Layout: row_ptr is u64[n+1] (row_ptr[0]=0, non-decreasing, row_ptr[n]=m); col is u32[m] with
 *     col[i] < n (Table II sizes imply 8-byte offsets and 4-byte IDs). Paths
 *     are row-major u32[W][stride]; row w holds path vertices 0..length[w]-1, then 0xFFFFFFFF.
 */
#ifndef LT_H
#define LT_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct lt_ctx lt_ctx;

typedef enum {
  LT_OK = 0,
  LT_ERR_INVALID = 1, /* bad argument: malformed CSR, start >= n, P == 0 or P > n, bad l/alpha */
  LT_ERR_STATE = 2,   /* call out of order */
  LT_ERR_OOM = 3,     /* device memory reservation failed (create / graph_load / walks_init) */
  LT_ERR_CUDA = 4,    /* a CUDA runtime error, or a device-side invariant violation */
  LT_ERR_NCCL = 5     /* reserved: the library issues no collective itself (the caller's torch.distributed
                         does, dist.py), so it never returns this */
} lt_status;

typedef enum {
  LT_APP_DEEPWALK = 0, /* uniform sampling, fixed length l */
  LT_APP_PPR = 1,      /* personalized PageRank: stop with probability alpha per step */
  LT_APP_PAGERANK = 2  /* PageRank / random walk with restart: fixed length l; at each step, with
                          probability p, restart at a uniform random vertex instead of moving to a
                          uniform neighbour (reading R23). Started with
                          lt_walks_init_pagerank (it takes both l and p). */
} lt_app;

typedef enum {
  /* Partition scheduling policy; Table III's four columns.
   * Resident mode uses only the order: selective = descending pending walks, else ID order.
   * Out-of-core mode: selective = load the partition with the most walks and evict the resident one
   * with the fewest; preemptive = run ready resident partitions while a load is in
   * flight; round robin = load in ID order, evict FIFO, no preemption. */
  LT_POLICY_SELECTIVE = 0,        /* PS + SS (LightTraffic's default) */
  LT_POLICY_ROUND_ROBIN = 1,      /* baseline: round robin + FIFO */
  LT_POLICY_SELECTIVE_ONLY = 2,   /* SS */
  LT_POLICY_PREEMPTIVE_ONLY = 3   /* PS with round-robin loading + FIFO eviction */
} lt_policy;

typedef enum {
  LT_INSERT_WARP_AGGREGATED = 0, /* __match_any_sync groups: one atomic per (warp, dest) */
  LT_INSERT_DIRECT = 1           /* one global atomic per walk ("direct write") */
} lt_insert_mode;

typedef enum {
  LT_LAYOUT_AUTO = 0, /* ADJ when 16 B x m fits in half of the free device memory and in the 64 GiB
                         a random gather can span at full rate on B200 (address-translation reach,
                         measured), else ADJ12 under the same two limits (when it applies), else CSR */
  LT_LAYOUT_CSR = 1,  /* steps gather row_ptr[v], row_ptr[v+1] and col[row_ptr[v] + i] */
  LT_LAYOUT_ADJ = 2,  /* steps gather adj[row_ptr[v] + i] = {u, deg(u), row_ptr[u]}: one access per step */
  LT_LAYOUT_ADJ12 = 3 /* the same in 12 B per entry {u, row_ptr[u] (40 bits), deg(u) (24 bits)}: needs
                         m < 2^40 and every degree < 2^24 (else LT_ERR_INVALID at load)
                         With ADJ / ADJ12 the steps never read col: a col the library copied is freed
                         at load, and a borrowed device col is not read after lt_graph_load_device
                         returns (the caller may free it). */
} lt_layout;

typedef struct lt_config {
  int device;                 /* CUDA ordinal */
  void* stream;               /* cudaStream_t to run on; NULL -> the legacy default stream */
  uint32_t chunk_walks;       /* C, walks per pool chunk, power of two >= 64; 0 -> 8192 */
  uint32_t ppr_max_len;       /* L_max, PPR step cap (reading R6); 0 -> 127 */
  uint32_t policy;            /* lt_policy */
  uint32_t insert_mode;       /* lt_insert_mode */
  uint32_t timing;            /* 1 -> CUDA events around every update launch (lt_stats.update_ms) */
  uint32_t block_threads;     /* update kernel block size (multiple of 32); 0 -> 256 */
  uint32_t blocks_per_sm;     /* update kernel resident blocks per SM for the grid; 0 -> occupancy */
  uint32_t l2_fetch_bytes;    /* cudaLimitMaxL2FetchGranularity set at create: 0 -> 32 (random
                                 sector gathers); 0xFFFFFFFF -> leave the device limit untouched */
  uint32_t gather_mode;       /* L2 hints of the CSR gathers: 0 none, 1 col evict_first, 2 +row_ptr
                                 evict_last, 3 col evict_first + L2::64B
                                 ...; lt_config_default sets 3 */
  uint32_t ilp;               /* walks advanced in lockstep per lane: 1, 2 or 4; 0 -> auto (1 with
                                 the ADJ layout, 2 with CSR: the measured best) */
  uint32_t layout;            /* lt_layout of the device graph the steps gather from */
  uint32_t path_mode;         /* 0: path entries buffered and written as full 32-B sectors;
                                 1: one 4-B store per step; 2: ABLATION, no path stores (paths
                                 invalid; lengths and stats still exact) */
  uint32_t zero_copy;         /* out-of-core: 1 -> adaptive zero copy when alpha*w < S_p */
  uint32_t zc_alpha_bytes;    /* alpha, bytes per walk; 0 -> 256 */
  uint32_t ooc_prefetch;      /* out-of-core: 1 -> before computing the selected partition, start loading the
                                 non-resident partition with the most walks into another block so the host
                                 link stays busy during the compute (parity-neutral); 0 -> off */
  uint64_t graph_pool_bytes;  /* 0 -> HBM-resident graph; > 0 -> out-of-core: the CSR stays in pinned
                                 host memory and a device graph pool of this many bytes caches
                                 partitions. Every partition must fit one block
                                 (block = the largest partition's CSR slice). */
  uint32_t rank, world;       /* range ownership across ranks (see lt_exchange_pack); world 0/1 -> off */
  uint32_t refill;            /* lane refill in the update kernel: 0 auto (on when P <= 16, or with at most
                                 64 buckets where its sorted flush applies: the measured best), 1 off (the
                                 batch kernel), 2 on */
  uint32_t visit_counts;      /* 1 -> count per-vertex visit frequency ("the visit
                                 frequency of each vertex is recorded") into a u64[n] device array
                                 reserved at lt_walks_init* and zeroed there: every path entry (start
                                 included) adds 1 to its vertex. Read with lt_get_visit_counts*. The
                                 kernels count in u32 while no count can reach 2^32 (W * stride <
                                 2^32) and widen at the end of lt_run — with the ADJ layout the 2^24 - 1
                                 highest-degree vertices count in slots packed by degree rank (the ADJ
                                 entry carries the slot; lt_stats.visit_hot_slots), otherwise with an
                                 augmented layout in
                                 16-bit halves for the vertices below a hub degree (lt_stats.hub_deg),
                                 a wrap detected exactly and recounted from the paths (an error under
                                 path_mode 2); 2 -> always count in u64. */
  uint32_t continue_resident; /* out-of-core: 1 -> a walk leaving the launched partition for another
                                 partition resident in the graph pool keeps stepping there instead of
                                 being appended to its bucket (parity-neutral);
                                 uses the lane-refill kernel. Ignored when the graph is HBM-resident. */
  uint32_t walk_spill;        /* with walk_pool_walks < W: 0 -> walk admission (below); 1 -> spill: every
                                 walk exists from the start and the walk pool EVICTS whole chunks of the
                                 buckets with the fewest pending walks to pinned host memory when it is
                                 full, and loads a partition's evicted chunks back before the partition
                                 is computed (reading R17). The copies are
                                 kernels reading / writing a pinned, mapped host store (no per-chunk
                                 cudaMemcpy). Single-rank contexts only. Paths are unchanged. */
  uint64_t walk_pool_walks;   /* m_w, the walk pool's capacity in walks (D4; SURVEY.md
                                 8(f) f3): 0 -> sized for all W walks. When W > m_w the walks are
                                 admitted in index order as the pool drains: lt_walks_init creates the
                                 first m_w, and the scheduler admits more whenever walks have ended, so
                                 at most m_w walks are ever live and the pool holds 2 m_w records
                                 (+ per-bucket slack) however large W is. Single-rank contexts only.
                                 Paths are unchanged. */
  uint32_t direct_start;      /* 0 auto: with one partition, one rank, an HBM-resident graph and no walk
                                 pool cap, lt_walks_init writes no walk records: the update kernel
                                 takes walk j straight from starts[j] (device starts must then stay
                                 valid until lt_run returns, as with walk admission); 1 -> off (records
                                 always built by the init kernel). Parity-neutral. */
  uint32_t l2_persist;        /* L2 set-aside for the lines the kernels tag evict_last (visit counters,
                                 row_ptr): 0 -> leave cudaLimitPersistingL2CacheSize as it is; 1 -> set
                                 it to the device maximum at lt_create (process-wide device state) */
  void* arena;                /* caller-owned device memory (e.g. a torch tensor) on cfg->device, or NULL
                                 (SURVEY.md §8(b)): when given, every pool the library reserves — graph,
                                 augmented adjacency, walk pool, paths, lengths, counters, staging — is
                                 sub-allocated from it (256-B aligned bump allocation; LT_ERR_OOM when it
                                 runs out), nothing is freed back, and each lt_graph_load* starts it over.
                                 It stays owned by the caller and must outlive the context. Not used for
                                 buffers shared through CUDA IPC (lt_exchange_buffers; lt_paths_buffers is
                                 refused) nor for the temporaries of lt_get_paths_rows. */
  uint64_t arena_bytes;
  uint32_t ooc_compress;      /* out-of-core: 0 auto -> a partition copied into the graph pool travels as
                                 compressed column blocks (32 entries: first value + zigzag deltas
                                 bit-packed at the block's width), expanded by a decode kernel on the
                                 load stream; partitions that would not shrink travel raw. Built once by
                                 lt_graph_load* (host threads). 1 -> off (raw CSR slices). The graph the
                                 steps read is identical either way (DESIGN.md §7 "Compressed partition
                                 transfers"). */
} lt_config;

typedef struct lt_stats {
  uint64_t num_walks;          /* W of the last lt_walks_init */
  uint64_t steps;              /* sum over walks of (path vertices - 1) ("steps") */
  uint64_t visits;             /* walk records consumed by update launches (residences) */
  uint64_t truncated;          /* PPR walks stopped by L_max */
  uint64_t sweeps;             /* scheduler passes over the partitions */
  uint64_t update_launches;    /* walk-update kernel launches in the last lt_run */
  uint64_t kernel_launches;    /* all kernels the library launched in the last lt_walks_init + lt_run */
  uint64_t chunks_total;       /* pool size in chunks */
  uint64_t chunks_free_min;    /* low-water mark of free chunks seen at sweep boundaries */
  uint64_t h2d_bytes;          /* host->device bytes moved by the last init/run/get calls */
  uint64_t d2h_bytes;
  double update_ms;            /* sum of CUDA-event durations of update launches (if timing) */
  double run_ms;               /* CUDA-event duration of the last lt_run (first launch..last) */
  double init_ms;              /* CUDA-event duration of the last lt_walks_init* */
  double graph_prep_ms;        /* device-side graph preparation in the last lt_graph_load* (ADJ build) */
  uint32_t layout;             /* lt_layout in use (LT_LAYOUT_CSR or LT_LAYOUT_ADJ) */
  uint32_t out_of_core;        /* 1 if the graph is host-resident with a device graph pool */
  /* out-of-core scheduler counters of the last lt_run (Table III) */
  uint64_t iterations;         /* partitions selected by scheduler.iteration() */
  uint64_t explicit_copies;    /* partitions copied into the graph pool */
  uint64_t pool_hits;          /* selections whose partition was already resident */
  uint64_t zero_copy_launches; /* selections served through zero copy */
  uint64_t preemptive_launches;/* ready partitions run while a load was in flight */
  uint64_t graph_h2d_bytes;    /* CSR bytes copied host -> device by the scheduler */
  uint64_t pool_blocks;        /* m_g */
  uint64_t pool_block_bytes;
  uint64_t admissions;         /* walk admissions (lt_walks_init's included) in the last init + run */
  uint64_t peak_live;          /* most live walks seen at a scheduler step */
  uint64_t direct_start;       /* 1 if the last lt_walks_init* used the direct start (no walk records) */
  uint64_t graph_device_bytes; /* device bytes of the graph the steps gather from: row_ptr + the CSR
                                  (layout CSR) or augmented (ADJ / ADJ12) entries of the owned
                                  vertices (all vertices when world == 1);
                                  0 out of core (see pool_blocks x pool_block_bytes) */
  uint64_t l2_persist_bytes;   /* cudaLimitPersistingL2CacheSize set at lt_create (lt_config.l2_persist) */
  uint64_t prefetches;         /* out-of-core loads started ahead of the selection (lt_config.ooc_prefetch) */
  /* walk spill (lt_config.walk_spill) in the last lt_walks_init + lt_run */
  uint64_t spilled_chunks;     /* walk-pool chunks evicted to pinned host memory */
  uint64_t reloaded_chunks;    /* evicted chunks loaded back before their partition was computed */
  uint64_t spill_d2h_bytes;    /* walk records moved device -> host by evictions */
  uint64_t spill_h2d_bytes;    /* walk records moved host -> device by reloads */
  uint64_t host_chunks_peak;   /* most chunks held in host memory at once */
  uint64_t spill_prefetched_chunks; /* reloads started during the previous partition's launch (overlapped) */
  /* per-phase breakdown of the last lt_run (update vs reshuffle vs loading). The
     reshuffle (bucket insertion, a5) is fused into the update kernels, so update_ms covers both. With
     lt_config.timing: */
  double load_ms;              /* graph-partition H2D copies on the load stream (out-of-core) */
  double spill_xfer_ms;        /* walk-spill copy kernels (evictions + reloads over PCIe) */
  uint64_t host_syncs;         /* scheduler round trips: count reads that wait for the device */
  uint64_t arena_bytes_used;   /* high-water mark of the caller arena (lt_config.arena), 0 without one */
  /* visit counting (lt_config.visit_counts = 1) of the last lt_walks_init + lt_run */
  uint64_t hub_deg;            /* 0: u32/u64 counters; > 0: paired 16-bit counters for vertices of degree
                                  < hub_deg, u32 for the rest (chosen at lt_walks_init) */
  uint64_t visit_recounts;     /* 1 if a 16-bit counter wrapped and the counts were recomputed from the
                                  paths at the end of lt_run (exact either way) */
  uint64_t graph_h2d_raw_bytes;/* out-of-core: CSR bytes of the partitions copied (graph_h2d_bytes is what
                                  crossed the link: smaller with lt_config.ooc_compress) */
  uint64_t ooc_compressed_bytes;/* out-of-core: host bytes of the compressed column blocks (0: off) */
  uint64_t visit_hot_slots;    /* visit counting with the ADJ layout: vertices whose counters are packed by
                                  degree rank (0: not used; then hub_deg tells the mode) */
} lt_stats;

/* Fill *cfg with defaults (device 0, legacy stream, C=8192, L_max=127, selective, aggregated,
 * gather_mode 3, ilp auto, layout auto, buffered path stores). */
lt_status lt_config_default(lt_config* cfg);

/* Create a context on cfg->device. No graph or walk memory is reserved yet. */
lt_status lt_create(const lt_config* cfg, lt_ctx** out);
void lt_destroy(lt_ctx* ctx);
const char* lt_last_error(void);

/* Range partitioning. Host-only utility, no GPU needed:
 * bounds[0]=0 < bounds[1] < ... < bounds[P]=n; partition k = [bounds[k], bounds[k+1]); edges go
 * with their source. Bounds balance the CSR bytes cost(v) = 8 v + 4 row_ptr[v]:
 * bounds[k] = min{v : P cost(v) >= k cost(n)} (exact), then forced strictly increasing.
 * Requires 1 <= P <= n. */
lt_status lt_partition_bounds(uint32_t n, const uint64_t* row_ptr, uint32_t P, uint32_t* bounds);

/* Load the graph and partition it into P ranges (a1). lt_graph_load copies host arrays into
 * device memory the library owns; lt_graph_load_device BORROWS device arrays (no copy; the caller
 * keeps them alive and unchanged until lt_destroy or the next load). Validates the CSR (host
 * variant: full check; device variant: row_ptr checked on a host copy, col range checked on the
 * device). */
lt_status lt_graph_load(lt_ctx* ctx, uint32_t n, uint64_t m, const uint64_t* row_ptr,
                        const uint32_t* col, uint32_t num_partitions);
lt_status lt_graph_load_device(lt_ctx* ctx, uint32_t n, uint64_t m, const uint64_t* d_row_ptr,
                               const uint32_t* d_col, uint32_t num_partitions);
/* Partition bounds in use: bounds must hold P+1 entries (query P with bounds == NULL). */
lt_status lt_get_bounds(lt_ctx* ctx, uint32_t* bounds, uint32_t* P);

/* Create W walks (a2): walk i has ID first_walk_id + i (the Philox key counter), starts at
 * starts[i] < n, and is appended to the bucket of its start's partition. length_or_alpha is the
 * DeepWalk length l (a non-negative integer) or the PPR alpha in (0, 1). starts is host memory
 * (lt_walks_init; copied before the call returns) or device memory (lt_walks_init_ex with
 * starts_on_device = 1; borrowed: it must stay valid and unchanged until lt_run returns, because walk
 * admission and the direct start read it during the run). W < 2^32 - 1. */
lt_status lt_walks_init(lt_ctx* ctx, uint64_t num_walks, const uint32_t* starts, lt_app app,
                        double length_or_alpha, uint64_t seed);
lt_status lt_walks_init_ex(lt_ctx* ctx, uint64_t num_walks, const uint32_t* starts, int starts_on_device,
                           uint64_t first_walk_id, lt_app app, double length_or_alpha, uint64_t seed);

/* PageRank / random walk with restart ("at each step, a walk has a probability p to
 * restart at a random vertex, instead of uniformly selecting one of the neighbors"; reading R23):
 * walk i (ID first_walk_id + i) starts at starts[i] and takes exactly `length` steps (l >= 0 integer;
 * a dead end without a restart stops it early). At step t the PPR coin word x0 of blk(w,t,0) decides:
 * x0 < floor(p 2^32) -> the next vertex is Lemire(n) over the step's word stream (a uniform vertex);
 * otherwise a uniform neighbour as in DeepWalk. 0 < p < 1. Path stride l+1. Same ownership, errors and
 * state rules as lt_walks_init_ex. Combine with lt_config.visit_counts for the visit-frequency
 * estimate of PageRank (the paper's output for this application). */
lt_status lt_walks_init_pagerank(lt_ctx* ctx, uint64_t num_walks, const uint32_t* starts, int starts_on_device,
                                 uint64_t first_walk_id, uint32_t length, double restart_p, uint64_t seed);

/* Run the partition scheduler until every walk has terminated (a3-a7). Blocks the host. */
lt_status lt_run(lt_ctx* ctx);

/* Row stride of the path matrix: l+1 (DeepWalk) or L_max+1 (PPR). */
lt_status lt_path_stride(lt_ctx* ctx, uint32_t* stride);

/* Copy all paths (W x stride u32, row-major) and lengths (W u32, path vertices) to HOST buffers.
 * Either pointer may be NULL to skip it. */
lt_status lt_get_paths(lt_ctx* ctx, uint32_t* paths, uint32_t* lengths);
/* Copy the rows listed in host array rows[count] (local walk indices) to host paths[count x stride]
 * and lengths[count]. */
lt_status lt_get_paths_rows(lt_ctx* ctx, const uint64_t* rows, uint64_t count, uint32_t* paths,
                            uint32_t* lengths);
/* Copy all paths / lengths into caller-owned DEVICE buffers (same layout as lt_get_paths). */
lt_status lt_get_paths_device(lt_ctx* ctx, uint32_t* d_paths, uint32_t* d_lengths);

lt_status lt_get_stats(lt_ctx* ctx, lt_stats* out);

/* Ragged copy-out of all paths to HOST buffers: offsets[W+1] (u64; offsets[0] = 0 and
 * offsets[w+1] - offsets[w] = length[w]) and vertices (u32; walk w's path vertices at
 * [offsets[w], offsets[w+1])). vertices_capacity is in entries; *total receives offsets[W]. If it is
 * short the offsets are still written and LT_ERR_INVALID is returned. Suited to PPR, whose rows are
 * mostly padding (E[length] = 1/alpha of L_max+1 slots). Scratch device memory is reserved on the first
 * call (never inside lt_run). */
lt_status lt_get_paths_compact(lt_ctx* ctx, uint64_t* offsets, uint32_t* vertices, uint64_t vertices_capacity,
                               uint64_t* total);

/* Visit frequency (lt_config.visit_counts = 1): counts[v] = number of path entries equal
 * to v over the walks of the last lt_walks_init* (on this rank: the starts it kept and the steps it
 * took; the sum over ranks is the global count). counts is caller-owned u64[n], host (lt_get_visit_counts)
 * or device (lt_get_visit_counts_device). LT_ERR_STATE before lt_run or when counting was off. */
lt_status lt_get_visit_counts(lt_ctx* ctx, uint64_t* counts);
lt_status lt_get_visit_counts_device(lt_ctx* ctx, uint64_t* d_counts);

/* End-to-end sampling into HOST buffers with the copy-out overlapped: the same result as
 * lt_walks_init_ex(W, starts, host, first_walk_id, ...) + lt_run + lt_get_paths, computed in
 * `chunks` consecutive walk ranges (0 -> 8) with two device path buffers: while range c+1 is walked,
 * range c's paths and lengths stream to the host on a copy stream. paths is W x stride (stride as
 * lt_path_stride would report: l+1 or L_max+1), lengths W; both should be pinned for the copies to
 * overlap. Single-rank contexts only (world == 1). Stats afterwards cover all ranges. */
lt_status lt_run_to_host(lt_ctx* ctx, uint64_t num_walks, const uint32_t* starts, uint64_t first_walk_id,
                         lt_app app, double length_or_alpha, uint64_t seed, uint32_t* paths, uint32_t* lengths,
                         uint32_t chunks);

/* lt_run_to_host with the ragged layout of lt_get_paths_compact: offsets[W+1] and vertices
 * (capacity in entries; W * stride always suffices). Each walk range's offsets and packed vertices
 * stream to the host while the next range walks. */
lt_status lt_run_to_host_compact(lt_ctx* ctx, uint64_t num_walks, const uint32_t* starts, uint64_t first_walk_id,
                                 lt_app app, double length_or_alpha, uint64_t seed, uint64_t* offsets,
                                 uint32_t* vertices, uint64_t vertices_capacity, uint32_t chunks);

/* ---- Range ownership across GPUs (the north star's multi-GPU mode, not
 * in the paper). With cfg.world = R > 1, rank r owns partitions [floor(P r / R), floor(P (r+1) / R));
 * every rank calls every function with identical arguments. lt_walks_init keeps the walks whose
 * start partition this rank owns. lt_run advances local walks until no owned bucket holds a walk;
 * a walk whose next partition belongs to rank q is appended to send bucket q instead. The caller
 * then runs a superstep exchange (paper_conf_icde_xing0wxl23_b200/dist.py):
 *   lt_exchange_pack -> all-to-all of counts and 16-B records (NCCL via torch.distributed) ->
 *   lt_exchange_insert -> lt_run ... until the global count of live walks is 0.
 * Path rows then hold only the entries this rank wrote (others 0xFFFFFFFF) and lengths only the
 * walks that ended here (others 0): the merged result is the element-wise min of the paths and the
 * max of the lengths over ranks. Walk records carry walk indices, identical on every rank. */
/* Walks waiting in owned buckets (*local) and in the send bucket of each rank (outgoing[world]).
 * Reuses the counts lt_run read last when no walk has moved since (no device round trip), else
 * reads them (one small D2H + stream synchronisation). */
lt_status lt_pending(lt_ctx* ctx, uint64_t* local, uint64_t* outgoing);
/* Move every send bucket into d_send (device, 16-B records, grouped by destination rank in rank
 * order); counts[world] (host) receives the number of records per destination (0 for this rank).
 * LT_ERR_INVALID if capacity (records) is too small. Asynchronous: d_send is complete in the order
 * of the context's stream (a collective enqueued after this call on that stream sees it). */
lt_status lt_exchange_pack(lt_ctx* ctx, void* d_send, uint64_t capacity, uint64_t* counts);
/* Insert `count` received records (device memory, read in stream order; the caller keeps it alive
 * until the next synchronising call, e.g. lt_run) into the owned buckets. Asynchronous. */
lt_status lt_exchange_insert(lt_ctx* ctx, const void* d_recv, uint64_t count);

/* ---- Peer exchange: the same superstep without the pack kernel and the all-to-all. Each rank
 * allocates two receive buffers (superstep parity 0 / 1) of `capacity` 16-B records and two u64
 * cursors with lt_exchange_buffers, the ranks share their buffers (device pointers valid in this
 * process: CUDA IPC through lt_ipc_handle / lt_ipc_open across processes, the pointers themselves
 * within one), and lt_exchange_attach installs the table. From then on the update kernels append a
 * walk whose next partition rank q owns straight into rank q's receive buffer of the current parity
 * (peer stores over NVLink, one atomic per (warp, rank) on q's cursor), overlapping the transfer with
 * the walk steps. Superstep (dist.run_supersteps_p2p): lt_run -> lt_exchange_sent -> a sum over
 * ranks of the records sent (the barrier after which every buffer of this parity is complete; 0 ends
 * the loop) -> lt_exchange_take (insert what arrived, reset that cursor, flip the parity).
 * Every rank must take in every superstep so that the parities stay aligned. */
/* This rank's buffers: recv[e] (capacity records) and cursor[e] for e = 0, 1; cursor[1] is
 * cursor[0] + 256 bytes (one allocation; each cursor in its own 256-B block). Reallocated only when the capacity changes (not once attached).
 * Zeroed cursors. LT_ERR_INVALID if world < 2. */
lt_status lt_exchange_buffers(lt_ctx* ctx, uint64_t capacity, void** recv, void** cursor);
/* Install the tables recv[e * world + q], cursor[e * world + q] (host arrays of device pointers,
 * 2 * world each; entry q = rank must be this rank's own buffers). All ranks' capacities must match. */
lt_status lt_exchange_attach(lt_ctx* ctx, void* const* recv, void* const* cursor);
/* Records this rank appended to other ranks' buffers in the current superstep (from lt_run's last
 * count read). LT_ERR_INVALID if a receive buffer overflowed. */
lt_status lt_exchange_sent(lt_ctx* ctx, uint64_t* sent);
/* After every rank's lt_run of this superstep has completed (the caller's collective): insert the
 * records that arrived in this rank's buffer of the current parity into the owned buckets, reset its
 * cursor and the sent count, flip the parity. *received = the number inserted. Stream-ordered. */
lt_status lt_exchange_take(lt_ctx* ctx, uint64_t* received);
/* One fused superstep of the peer exchange, with no host synchronisation (one owned partition per
 * rank, HBM-resident, no walk-pool cap): insert the walks peers appended in the previous superstep
 * (count read on the device), reset that cursor, advance every owned walk in one update launch (walks
 * end or are appended to their owner's buffer of this superstep's parity), write the number of records
 * this rank sent to *d_sent (device u64), flip the parity. Loop (dist.run_supersteps_p2p_fused):
 * lt_superstep_p2p -> sum of d_sent over ranks (a device all-reduce; 0 ends it) -> ..., then one
 * lt_run to finalise statistics and visit counts. */
lt_status lt_superstep_p2p(lt_ctx* ctx, unsigned long long* d_sent);
/* Paths on one rank (range ownership; "the merged result lands on rank 0"): every rank
 * writes its path entries and lengths straight into the HOME rank's path matrix and length array over
 * peer memory (NVLink; stores buffered into 32-B sectors as usual), so when the last superstep ends the
 * home rank holds every walk's path — no cross-rank merge, and the other ranks keep no path matrix of
 * their own from their next lt_walks_init on (the home's capacity is checked there).
 * lt_paths_buffers (home rank, after its lt_walks_init): its matrix, length array and the matrix capacity
 * in u32 entries, for sharing (CUDA IPC through lt_ipc_handle / lt_ipc_open across processes, the
 * pointers themselves between threads). lt_paths_attach (every other rank): install the home's buffers,
 * or NULL, NULL to write locally again; with path_mode 1 it must precede lt_walks_init (which stores
 * path[w][0]), with path_mode 0 it may follow it. In the epoch of the first lt_paths_buffers call the
 * home's lt_walks_init has pre-filled its matrix: every rank's writes must start after it (dist.py
 * synchronises and barriers once). From then on the home's lt_walks_init neither pre-fills nor zeroes
 * its matrix and lengths (every length is written once per epoch where the walk ends; rows are padded
 * lazily by the first copy-out), so later epochs need no barrier. lt_get_paths* on an attached rank:
 * LT_ERR_STATE. */
lt_status lt_paths_buffers(lt_ctx* ctx, void** d_paths, void** d_lengths, uint64_t* capacity_entries);
lt_status lt_paths_attach(lt_ctx* ctx, void* d_paths, void* d_lengths, uint64_t capacity_entries);
/* CUDA IPC of a device allocation's base pointer (handle: 64 bytes), and opening another process's
 * handle on this context's device (closed at lt_destroy). */
lt_status lt_ipc_handle(const void* dptr, void* handle);
lt_status lt_ipc_open(lt_ctx* ctx, const void* handle, void** dptr);

/* Diagnostic (SURVEY.md §4 pin P2): the update kernels' Philox4x32-10 (reading R3) evaluated on the
 * device for n counters ctr[4i..4i+3] and keys key[2i..2i+1] (host arrays), out[4i..4i+3] = the block.
 * Lets tests compare the device RNG with cuRAND's curand_Philox4x32_10. Synchronous. */
lt_status lt_philox_device(int device, uint64_t n, const uint32_t* ctr, const uint32_t* key, uint32_t* out);

/* The compressed-partition format of lt_config.ooc_compress (host encoder, for tests and tools; no GPU):
 * col[0, len) is cut into blocks of 32 entries; block j is hdr[2j] = its first value, hdr[2j+1] = the offset
 * of its payload in words; its width w = hdr[2(j+1)+1] - hdr[2j+1] (hdr holds ceil(len/32) + 1 entries, the
 * last a sentinel); bits [i w, (i+1) w) of its payload (little-endian within words) hold entry i's zigzag-
 * coded difference (col[i] - col[i-1]) mod 2^32 for i = 1..31 (entry 0 codes 0). *words receives the payload
 * length; with pay == NULL only that is computed. Caller-owned host buffers. */
lt_status lt_compress_columns(const uint32_t* col, uint64_t len, uint32_t* hdr, uint32_t* pay, uint64_t* words);

/* Walk-pool invariants (a6), for tests and debugging; synchronizes the stream. Conservation:
 * pending + finished == num_walks; free_chunks + ring_chunks == total_chunks. */
typedef struct lt_pool_state {
  int64_t free_chunks;     /* free-stack depth */
  uint64_t ring_chunks;    /* installed (non-empty) ring slots over all partitions */
  uint64_t host_chunks;    /* chunks evicted to host memory (walk spill) */
  uint64_t total_chunks;
  uint64_t pending;        /* sum over partitions of cursor - head (walks waiting in buckets) */
  uint64_t finished;       /* walks with a recorded length */
  uint32_t device_err;     /* device error bits (1: pool exhausted, 2: ring slot reinstalled) */
  uint32_t reserved;
} lt_pool_state;
lt_status lt_get_pool_state(lt_ctx* ctx, lt_pool_state* out);

#ifdef __cplusplus
}
#endif
#endif
