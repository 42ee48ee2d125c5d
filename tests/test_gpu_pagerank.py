"""GPU parity for SURVEY.md §8(f) f2: PageRank as a random walk with restart, plus per-vertex visit
frequency (§IV-A "PageRank ... at each step, a walk has a probability p to restart at a
random vertex, instead of uniformly selecting one of the neighbors"; reading R23).

Paths and visit counts are integer data: the bar is exact equality with the CPU oracle, walk by walk
and vertex by vertex, for every partition count, kernel variant, residency mode and rank count.
"""
import threading

import numpy as np
import pytest

import lt_inputs
import oracle as O
import paper_conf_icde_xing0wxl23_b200 as LT
from paper_conf_icde_xing0wxl23_b200 import dist as ltdist

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def cfg1():
    """BASELINE.json configs[0]'s graph: R-MAT scale 12, 65,536 tuples."""
    return lt_inputs.rmat_cpu(12, 65_536, seed=1)


def gpu_pagerank(g, starts, length, p, seed, P, first=0, **cfg):
    cfg.setdefault("visit_counts", True)
    with LT.Engine(**cfg) as e:
        e.graph_load(g.row_ptr, g.col, P)
        e.walks_init_pagerank(starts, length, p, seed, first)
        e.run()
        paths, lengths = e.get_paths()
        return paths, lengths, e.visit_counts(), e.stats()


def oracle_pagerank(g, starts, length, p, seed, first=0):
    ids = np.arange(first, first + len(starts), dtype=np.uint64)
    return O.walks(g.row_ptr, g.col, starts, app=O.PAGERANK, length=length, alpha=p, seed=seed, ids=ids)


def assert_pagerank_parity(g, starts, length, p, seed, P, first=0, **cfg):
    paths, lengths, counts, st = gpu_pagerank(g, starts, length, p, seed, P, first=first, **cfg)
    op, ol, osteps, _ = oracle_pagerank(g, starts, length, p, seed, first=first)
    np.testing.assert_array_equal(lengths, ol)
    np.testing.assert_array_equal(paths, op)
    assert st["steps"] == osteps
    np.testing.assert_array_equal(counts, O.visit_counts(op, ol, g.n))
    return paths, counts, st


@pytest.mark.parametrize("p", [0.15, 0.5, 0.999])
@pytest.mark.parametrize("P", [1, 4, 64])
def test_pagerank_exact(gpu, cfg1, p, P):
    starts = lt_inputs.deepwalk_starts(4096, cfg1.n)
    paths, counts, st = assert_pagerank_parity(cfg1, starts, 20, p, 7, P)
    assert counts.sum() == 4096 * 21  # no dead ends after preprocessing: every walk has l+1 entries
    if P > 1:  # restarts land anywhere: walks change partition through restarts as well as edges
        assert st["visits"] > 4096


@pytest.mark.parametrize("layout", [LT.LAYOUT_CSR, LT.LAYOUT_ADJ, LT.LAYOUT_ADJ12])
@pytest.mark.parametrize("ilp,refill", [(1, 1), (2, 1), (4, 1), (1, 2)])
@pytest.mark.parametrize("P", [1, 8])
@pytest.mark.parametrize("width", [1, 2])  # u32 counters (auto) / forced u64 counters
def test_pagerank_kernel_variants(gpu, cfg1, layout, ilp, refill, P, width):
    starts = lt_inputs.deepwalk_starts(3000, cfg1.n)
    assert_pagerank_parity(cfg1, starts, 17, 0.3, 11, P, layout=layout, ilp=ilp, refill=refill, chunk_walks=256,
                           visit_counts=width)


def test_pagerank_restarts_cross_partitions_and_first_walk_id(gpu, cfg1):
    starts = lt_inputs.ppr_starts(5000, cfg1.argmax_deg)  # all from the hub: restarts spread them
    assert_pagerank_parity(cfg1, starts, 9, 0.25, 3, P=16, first=123_456_789_012)


@pytest.mark.parametrize("W", [0, 1, 33])
def test_pagerank_ragged_and_zero_length(gpu, cfg1, W):
    starts = lt_inputs.deepwalk_starts(W, cfg1.n)
    assert_pagerank_parity(cfg1, starts, 5, 0.2, 1, P=3)
    assert_pagerank_parity(cfg1, lt_inputs.deepwalk_starts(40, cfg1.n), 0, 0.2, 1, P=3)


def test_pagerank_dead_end_restart(gpu):
    """A vertex with no edges: without a restart the walk stops there (reading R9), a restart still
    leaves it (the coin is tossed before the degree is looked at, reading R23)."""
    g = lt_inputs.small_graph([(0, 1), (1, 2)], n=4)  # vertex 3 is isolated
    starts = np.full(2000, 3, dtype=np.uint32)
    paths, counts, _ = assert_pagerank_parity(g, starts, 6, 0.5, 9, P=2)
    lengths = (paths != O.EMPTY).sum(axis=1)
    assert lengths.min() == 1 and lengths.max() == 7


@pytest.mark.parametrize("app,param", [(LT.DEEPWALK, 12), (LT.PPR, 0.15)])
@pytest.mark.parametrize("P", [1, 5])
def test_visit_counts_other_apps(gpu, cfg1, app, param, P):
    starts = lt_inputs.deepwalk_starts(4096, cfg1.n) if app == LT.DEEPWALK else lt_inputs.ppr_starts(4096, cfg1.argmax_deg)
    with LT.Engine(visit_counts=True) as e:
        e.graph_load(cfg1.row_ptr, cfg1.col, P)
        e.walks_init(starts, app, param, 5)
        e.run()
        counts = e.visit_counts()
    kw = dict(app=O.DEEPWALK, length=int(param)) if app == LT.DEEPWALK else dict(app=O.PPR, alpha=param)
    op, ol, _, _ = O.walks(cfg1.row_ptr, cfg1.col, starts, seed=5, **kw)
    np.testing.assert_array_equal(counts, O.visit_counts(op, ol, cfg1.n))


def test_visit_counts_device_copy_and_epochs(gpu, cfg1):
    import torch
    starts = lt_inputs.deepwalk_starts(1000, cfg1.n)
    with LT.Engine(visit_counts=True) as e:
        e.graph_load(cfg1.row_ptr, cfg1.col, 2)
        for seed in (1, 2):  # counts are zeroed at every lt_walks_init*
            e.walks_init_pagerank(starts, 8, 0.15, seed)
            e.run()
            d = torch.zeros(cfg1.n, dtype=torch.int64, device="cuda")
            e.visit_counts(d)
            op, ol, _, _ = oracle_pagerank(cfg1, starts, 8, 0.15, seed)
            np.testing.assert_array_equal(d.cpu().numpy().view(np.uint64), O.visit_counts(op, ol, cfg1.n))


def test_visit_counts_errors(gpu, cfg1):
    starts = lt_inputs.deepwalk_starts(64, cfg1.n)
    with LT.Engine() as e:  # counting off
        e.graph_load(cfg1.row_ptr, cfg1.col, 1)
        e.walks_init_pagerank(starts, 4, 0.2, 1)
        e.run()
        with pytest.raises(LT.LTError) as ei:
            e.visit_counts()
        assert ei.value.status == 2  # LT_ERR_STATE
    with LT.Engine(visit_counts=True) as e:
        e.graph_load(cfg1.row_ptr, cfg1.col, 1)
        e.walks_init_pagerank(starts, 4, 0.2, 1)
        with pytest.raises(LT.LTError):
            e.visit_counts()  # before lt_run
        for bad in (0.0, 1.0, -0.1):
            with pytest.raises(LT.LTError) as ei:
                e.walks_init_pagerank(starts, 4, bad, 1)
            assert ei.value.status == 1
        with pytest.raises(LT.LTError) as ei:
            e.walks_init(starts, LT.PAGERANK, 4, 1)  # PageRank needs both l and p
        assert ei.value.status == 1


# ---- paired 16-bit visit counters with hub counters (VIS 3, DESIGN.md §7 "PageRank and visit counts")
def _deg(g):
    rp = g.row_ptr.astype(np.int64)
    return rp[1:] - rp[:-1]


@pytest.mark.parametrize("P,refill", [(1, 2), (1, 1), (8, 2), (8, 1)])
def test_visit_counts_16bit_halves_with_hubs(gpu, cfg1, P, refill):
    """VIS 3 (ADJ12): 65,536 PageRank walks of length 80 on configs[0]'s graph: 5.3M path entries over ~130K
    CSR entries put the hub degree near 100, so both counter kinds (16-bit halves, u32 hubs) and both halves
    of a word are exercised; counts equal the oracle's bincount vertex by vertex."""
    starts = lt_inputs.deepwalk_starts(65_536, cfg1.n)
    _, counts, st = assert_pagerank_parity(cfg1, starts, 80, 0.15, 21, P, layout=LT.LAYOUT_ADJ12, refill=refill)
    deg = _deg(cfg1)
    assert st["visit_hot_slots"] == 0
    assert 64 <= st["hub_deg"] < deg.max(), st["hub_deg"]
    hub = deg >= st["hub_deg"]
    assert hub.any() and (~hub).any()
    assert counts[hub].sum() > 0 and counts[~hub].sum() > 0
    assert st["visit_recounts"] == 0


@pytest.mark.parametrize("P,refill", [(1, 2), (1, 1), (8, 2), (8, 1)])
@pytest.mark.parametrize("app", ["pagerank", "deepwalk", "ppr"])
def test_visit_counts_degree_slots(gpu, cfg1, P, refill, app):
    """VIS 4 (ADJ): counters of the highest-degree vertices packed by degree rank, the slot carried by the
    ADJ entry; starts, restarts and unslotted vertices count per vertex. Exact against the oracle for
    every app, kernel and partition count."""
    if app == "pagerank":
        starts = lt_inputs.deepwalk_starts(20_000, cfg1.n)
        _, counts, st = assert_pagerank_parity(cfg1, starts, 30, 0.15, 5, P, layout=LT.LAYOUT_ADJ, refill=refill)
    else:
        starts = (lt_inputs.deepwalk_starts(20_000, cfg1.n) if app == "deepwalk"
                  else lt_inputs.ppr_starts(20_000, cfg1.argmax_deg))
        with LT.Engine(visit_counts=True, layout=LT.LAYOUT_ADJ, refill=refill) as e:
            e.graph_load(cfg1.row_ptr, cfg1.col, P)
            if app == "deepwalk":
                e.walks_init(starts, LT.DEEPWALK, 30, 5)
            else:
                e.walks_init(starts, LT.PPR, 0.15, 5)
            e.run()
            counts, st = e.visit_counts(), e.stats()
        kw = dict(app=O.DEEPWALK, length=30) if app == "deepwalk" else dict(app=O.PPR, alpha=0.15)
        op, ol, _, _ = O.walks(cfg1.row_ptr, cfg1.col, starts, seed=5, **kw)
        np.testing.assert_array_equal(counts, O.visit_counts(op, ol, cfg1.n))
    assert st["visit_hot_slots"] == cfg1.n and st["hub_deg"] == 0


def test_visit_counts_degree_slots_beyond_2_24(gpu):
    """More vertices than slots (n > 2^24 - 1): the lowest-degree vertices have no slot and count per
    vertex through the same kernel. R-MAT scale 26 with 400M tuples, 1M PageRank walks of length 20;
    exact against the oracle."""
    import torch
    g = lt_inputs.rmat_gpu(26, 400_000_000, seed=4)
    assert g.n > (1 << 24)
    rp, col = g.row_ptr.cpu().numpy().view(np.uint64), g.col.cpu().numpy().view(np.uint32)
    starts = lt_inputs.deepwalk_starts(1_000_000, g.n)
    with LT.Engine(visit_counts=True, layout=LT.LAYOUT_ADJ) as e:
        e.graph_load(g.row_ptr, g.col, 1)
        e.walks_init_pagerank(torch.from_numpy(starts.view(np.int32)).cuda(), 20, 0.15, 9)
        e.run()
        counts, st = e.visit_counts(), e.stats()
    op, ol, _, _ = O.walks(rp, col, starts, app=O.PAGERANK, length=20, alpha=0.15, seed=9)
    ref = O.visit_counts(op, ol, g.n)
    np.testing.assert_array_equal(counts, ref)
    assert st["visit_hot_slots"] == (1 << 24) - 1
    deg = np.diff(rp.astype(np.int64))
    unslotted = np.argsort(-deg, kind="stable")[(1 << 24) - 1:]
    assert ref[unslotted].sum() > 0


def test_visit_counts_csr_keeps_u32(gpu, cfg1):
    starts = lt_inputs.deepwalk_starts(2048, cfg1.n)
    _, _, st = assert_pagerank_parity(cfg1, starts, 10, 0.15, 2, 1, layout=LT.LAYOUT_CSR)
    assert st["hub_deg"] == 0 and st["visit_hot_slots"] == 0


@pytest.mark.parametrize("P", [1, 4])
def test_visit_counts_16bit_wrap_is_recounted(gpu, cfg1, P):
    """VIS 3 (ADJ12): 70,000 DeepWalk walks of length 3 all from one low-degree vertex: its count
    (>= 70,000) wraps its 16-bit half (and carries into the neighbour's half); the end-of-run sum check
    sees the shortfall and the counts are recomputed from the paths, exactly. VIS 4 (ADJ) counts the
    same run exactly with nothing to recount."""
    deg = _deg(cfg1)
    pos = np.flatnonzero(deg > 0)
    v0 = int(pos[np.argmin(deg[pos])])
    starts = np.full(70_000, v0, dtype=np.uint32)
    op, ol, _, _ = O.walks(cfg1.row_ptr, cfg1.col, starts, app=O.DEEPWALK, length=3, seed=4)
    ref = O.visit_counts(op, ol, cfg1.n)
    with LT.Engine(visit_counts=True, layout=LT.LAYOUT_ADJ12) as e:
        e.graph_load(cfg1.row_ptr, cfg1.col, P)
        e.walks_init(starts, LT.DEEPWALK, 3, 4)
        e.run()
        counts = e.visit_counts()
        st = e.stats()
    assert st["hub_deg"] > deg[v0] and st["visit_recounts"] == 1
    np.testing.assert_array_equal(counts, ref)
    assert counts[v0] >= 70_000
    with LT.Engine(visit_counts=True, layout=LT.LAYOUT_ADJ) as e:
        e.graph_load(cfg1.row_ptr, cfg1.col, P)
        e.walks_init(starts, LT.DEEPWALK, 3, 4)
        e.run()
        np.testing.assert_array_equal(e.visit_counts(), ref)
        assert e.stats()["visit_hot_slots"] > 0 and e.stats()["visit_recounts"] == 0
    # without paths there is nothing to recount from: a clear error, and u64 counters (visit_counts=2) work
    with LT.Engine(visit_counts=True, layout=LT.LAYOUT_ADJ12, path_mode=2) as e:
        e.graph_load(cfg1.row_ptr, cfg1.col, P)
        e.walks_init(starts, LT.DEEPWALK, 3, 4)
        with pytest.raises(LT.LTError) as ei:
            e.run()
        assert "wrapped" in str(ei.value)
    with LT.Engine(visit_counts=2, layout=LT.LAYOUT_ADJ12, path_mode=2) as e:
        e.graph_load(cfg1.row_ptr, cfg1.col, P)
        e.walks_init(starts, LT.DEEPWALK, 3, 4)
        e.run()
        np.testing.assert_array_equal(e.visit_counts(), ref)
        assert e.stats()["hub_deg"] == 0


@pytest.mark.parametrize("blocks", [1, 3])
@pytest.mark.parametrize("zero_copy", [False, True])
def test_pagerank_out_of_core(gpu, blocks, zero_copy):
    g = lt_inputs.rmat_cpu(14, 16 * 2 ** 14, seed=2)
    b = LT.partition_bounds(g.row_ptr, 16).astype(np.int64)
    rp = g.row_ptr.astype(np.int64)
    rpb = max(8 * (b[k + 1] - b[k] + 1) for k in range(16))
    colb = max(4 * (rp[b[k + 1]] - rp[b[k]]) for k in range(16))
    block = ((rpb + 255) // 256 * 256 + colb + 255) // 256 * 256  # one graph-pool block (lt_abi.cpp)
    starts = lt_inputs.deepwalk_starts(g.n, g.n)
    _, _, st = assert_pagerank_parity(g, starts, 10, 0.15, 4, 16, graph_pool_bytes=blocks * block,
                                      zero_copy=zero_copy)
    assert st["out_of_core"] == 1


@pytest.mark.parametrize("world", [2, 3])
@pytest.mark.parametrize("p2p", [False, True])
def test_pagerank_ownership_and_merged_visit_counts(gpu, world, p2p):
    """Range ownership with restarts: a restart may send a walk to any rank. Merged
    paths equal the oracle; visit counts summed over ranks equal the oracle's."""
    import torch
    g = lt_inputs.rmat_cpu(13, 8 * 2 ** 13, seed=3)
    starts = lt_inputs.deepwalk_starts(2 * g.n, g.n)
    hub = ltdist.ThreadComm.Hub(world)
    results, errors = [None] * world, []

    def rank_main(r):
        try:
            with LT.Engine(rank=r, world=world, visit_counts=True, chunk_walks=512) as e:
                e.graph_load(g.row_ptr, g.col, 12)
                e.walks_init_pagerank(starts, 12, 0.2, 6)
                comm = ltdist.ThreadComm(hub, r)
                if p2p:  # peer exchange: restarts send walks to any rank's receive buffer
                    ltdist.attach_peers(e, comm, len(starts))
                    ltdist.run_supersteps_p2p(e, comm, "cuda")
                else:
                    ltdist.run_supersteps(e, comm, "cuda")
                paths, lengths = ltdist.merge_paths(e, comm)
                counts = ltdist.merge_visit_counts(e, comm, "cuda")
                torch.cuda.synchronize()
                results[r] = (paths.cpu().numpy().view(np.uint32), lengths.cpu().numpy().view(np.uint32),
                              counts.cpu().numpy().view(np.uint64))
        except Exception as ex:
            errors.append(ex)
            hub.barrier.abort()

    th = [threading.Thread(target=rank_main, args=(r,)) for r in range(world)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    if errors:
        raise errors[0]
    op, ol, _, _ = oracle_pagerank(g, starts, 12, 0.2, 6)
    expect = O.visit_counts(op, ol, g.n)
    for paths, lengths, counts in results:
        np.testing.assert_array_equal(lengths, ol)
        np.testing.assert_array_equal(paths, op)
        np.testing.assert_array_equal(counts, expect)
