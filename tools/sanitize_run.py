#!/usr/bin/env python3
"""Small runs of every kernel path for compute-sanitizer (memcheck / racecheck / synccheck /
initcheck): resident P=1 (refill), P=4 (batch kernel, CSR and ADJ), PPR, out-of-core with zero copy,
two-rank ownership, streamed run_to_host (dense and ragged), ragged copy-out, PageRank with u32 / u64
visit counters, out-of-core continuation, walk admission, paths off, the direct start (P = 1, both
path modes, device starts), the compact ADJ12 layout, slice-only ownership (CSR / ADJ / ADJ12, host and
borrowed device graphs), the peer exchange (CSR / ADJ); round 2: O records through the lane-refill kernel at
P > 1 and the walk spill
(evict / reload kernels, tail-capped launches); second session: visit counters by degree slot and paired
16-bit counters with a forced wrap recount, compressed partition transfers (decode kernel)."""
import os
import sys
import threading

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import lt_inputs  # noqa: E402
import paper_conf_icde_xing0wxl23_b200 as LT  # noqa: E402
from paper_conf_icde_xing0wxl23_b200 import dist as ltdist  # noqa: E402

QUICK = "--quick" in sys.argv  # racecheck (shared-memory hazards) is slow: the kernels with shared staging only
g = lt_inputs.rmat_cpu(12, 65_536, seed=1)
starts = lt_inputs.deepwalk_starts(4096, g.n)
pstarts = lt_inputs.ppr_starts(4096, g.argmax_deg)
for kw in [dict(P=1), dict(P=4, layout=LT.LAYOUT_CSR), dict(P=4, layout=LT.LAYOUT_ADJ), dict(P=4, refill=2),
           dict(P=1, layout=LT.LAYOUT_ADJ12), dict(P=4, layout=LT.LAYOUT_ADJ12), dict(P=1, path_mode=1),
           dict(P=1, direct_start=False), dict(P=4, refill=2, layout=LT.LAYOUT_CSR)]:
    P = kw.pop("P")
    with LT.Engine(chunk_walks=256, **kw) as e:
        e.graph_load(g.row_ptr, g.col, P)
        for st, app, prm in [(starts, LT.DEEPWALK, 10), (pstarts, LT.PPR, 0.15)]:
            e.walks_init(st, app, prm, 1)
            e.run()
            e.get_paths()
# round 2: O records at P > 1 (lane refill) and walk spill
g14 = lt_inputs.rmat_cpu(14, 16 * 2 ** 14, seed=2)
s14 = lt_inputs.deepwalk_starts(4 * g14.n, g14.n)
with LT.Engine(chunk_walks=256, refill=2) as e:
    e.graph_load(g14.row_ptr, g14.col, 8)
    e.walks_init(s14, LT.DEEPWALK, 12, 1)
    e.run()
    e.get_paths()
with LT.Engine(chunk_walks=256, walk_pool_walks=len(s14) // 5, walk_spill=True) as e:
    e.graph_load(g14.row_ptr, g14.col, 8)
    e.walks_init(s14, LT.DEEPWALK, 12, 1)
    e.run()
    e.get_paths()
if QUICK:  # racecheck: the kernels with shared-memory staging (lane refill at P = 1 / P > 1, batch, spill)
    print("sanitize_run done")
    raise SystemExit(0)
with LT.Engine(graph_pool_bytes=1 << 20, zero_copy=True, chunk_walks=256) as e:
    e.graph_load(g.row_ptr, g.col, 8)
    e.walks_init(starts, LT.DEEPWALK, 10, 1)
    e.run()
    e.get_paths()
with LT.Engine() as e:
    e.graph_load(g.row_ptr, g.col, 1)
    e.run_to_host(starts, LT.DEEPWALK, 10, 1, chunks=3)
    e.run_to_host_compact(pstarts, LT.PPR, 0.15, 1, chunks=3)
    e.walks_init(pstarts, LT.PPR, 0.15, 2)
    e.run()
    e.get_paths_compact()
# PageRank with fused visit counters (u32 and u64), the CSR and ADJ layouts, P = 1 and P = 4
# (round 2, second session: ADJ -> counters by degree slot, ADJ12 -> paired 16-bit counters)
for kw in [dict(P=1, visit_counts=1), dict(P=4, visit_counts=2, layout=LT.LAYOUT_CSR), dict(P=4, visit_counts=1),
           dict(P=1, visit_counts=1, layout=LT.LAYOUT_ADJ12), dict(P=4, visit_counts=1, layout=LT.LAYOUT_ADJ12)]:
    P = kw.pop("P")
    with LT.Engine(chunk_walks=256, **kw) as e:
        e.graph_load(g.row_ptr, g.col, P)
        e.walks_init_pagerank(starts, 10, 0.2, 1)
        e.run()
        e.get_paths()
        e.visit_counts()
# a forced 16-bit wrap recounted from the paths (k_widen16 + k_recount)
with LT.Engine(visit_counts=1, layout=LT.LAYOUT_ADJ12) as e:
    e.graph_load(g.row_ptr, g.col, 1)
    e.walks_init(np.full(70_000, int(np.flatnonzero(np.diff(g.row_ptr.astype(np.int64)) > 0)[-1]), dtype=np.uint32),
                 LT.DEEPWALK, 3, 4)
    e.run()
    e.visit_counts()
# compressed partition transfers (k_decode_cols) with and without zero copy, P = 16
for zc in (False, True):
    with LT.Engine(graph_pool_bytes=1 << 20, zero_copy=zc, chunk_walks=256, ooc_compress=True) as e:
        e.graph_load(g14.row_ptr, g14.col, 16)
        e.walks_init(s14[:4096], LT.DEEPWALK, 10, 1)
        e.run()
        e.get_paths()
# out of core with continuation into resident partitions, and walk admission under a pool cap
with LT.Engine(graph_pool_bytes=1 << 20, zero_copy=True, continue_resident=True, chunk_walks=256,
               walk_pool_walks=1000) as e:
    e.graph_load(g.row_ptr, g.col, 8)
    e.walks_init(starts, LT.DEEPWALK, 10, 1)
    e.run()
    e.get_paths()
with LT.Engine(path_mode=2, walk_pool_walks=500, chunk_walks=64, visit_counts=True) as e:
    e.graph_load(g.row_ptr, g.col, 3)
    e.walks_init_pagerank(starts, 10, 0.2, 1)
    e.run()
    e.get_paths(paths=False)
import torch  # noqa: E402

with LT.Engine() as e:  # direct start from device starts
    e.graph_load(g.row_ptr, g.col, 1)
    e.walks_init(torch.from_numpy(starts.view(np.int32)).cuda(), LT.DEEPWALK, 10, 1)
    e.run()
    e.get_paths()
d_rp = torch.from_numpy(g.row_ptr.view(np.int64)).cuda()
d_col = torch.from_numpy(g.col.view(np.int32)).cuda()
for layout, device_graph in [(LT.LAYOUT_AUTO, False), (LT.LAYOUT_CSR, False), (LT.LAYOUT_ADJ12, False),
                             (LT.LAYOUT_ADJ, True), (LT.LAYOUT_CSR, True)]:
    hub = ltdist.ThreadComm.Hub(2)

    def rank(r):
        with LT.Engine(rank=r, world=2, chunk_walks=256, layout=layout) as e:
            if device_graph:
                e.graph_load(d_rp, d_col, 4)
            else:
                e.graph_load(g.row_ptr, g.col, 4)
            e.walks_init(starts, LT.DEEPWALK, 10, 1)
            comm = ltdist.ThreadComm(hub, r)
            ltdist.run_supersteps(e, comm, "cuda")
            ltdist.merge_paths(e, comm)

    th = [threading.Thread(target=rank, args=(r,)) for r in range(2)]
    for t in th:
        t.start()
    for t in th:
        t.join()
# peer exchange (walks appended into the owner's receive buffer by the update kernels), CSR and ADJ
for layout in (LT.LAYOUT_CSR, LT.LAYOUT_ADJ):
    hub = ltdist.ThreadComm.Hub(2)

    def rank_p2p(r):
        with LT.Engine(rank=r, world=2, chunk_walks=256, layout=layout) as e:
            e.graph_load(g.row_ptr, g.col, 4)
            e.walks_init(starts, LT.DEEPWALK, 10, 1)
            comm = ltdist.ThreadComm(hub, r)
            ltdist.attach_peers(e, comm, len(starts))
            ltdist.run_supersteps_p2p(e, comm, "cuda")
            ltdist.merge_paths(e, comm)

    th = [threading.Thread(target=rank_p2p, args=(r,)) for r in range(2)]
    for t in th:
        t.start()
    for t in th:
        t.join()
print("sanitize_run done")
