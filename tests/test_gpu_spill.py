"""Walk spill (SURVEY.md §8(f) f3 and the walk-chunk side of §8(a) a8): with lt_config.walk_spill and a walk
pool smaller than the walk set, every walk exists from the start, the pool evicts whole chunks of the
buckets with the fewest pending walks to pinned host memory when it is full, and loads a partition's
evicted chunks back before computing it (reading R17). Paths, lengths and
visit counts must equal the oracle bit-exactly whatever the cap, partition count, kernel, scheduling policy,
chunk size and residency mode; every evicted chunk comes back, and the pool's conservation holds."""
import numpy as np
import pytest

import lt_inputs
import oracle as O
import paper_conf_icde_xing0wxl23_b200 as LT

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def g14():
    return lt_inputs.rmat_cpu(14, 16 * 2 ** 14, seed=2)


def oracle_for(g, starts, app, param, seed, length):
    if app == LT.DEEPWALK:
        return O.walks(g.row_ptr, g.col, starts, app=O.DEEPWALK, length=length, seed=seed)
    if app == LT.PPR:
        return O.walks(g.row_ptr, g.col, starts, app=O.PPR, alpha=param, seed=seed)
    return O.walks(g.row_ptr, g.col, starts, app=O.PAGERANK, length=length, alpha=param, seed=seed)


def run_spill(g, starts, app, param, seed, P, cap, length=15, **cfg):
    with LT.Engine(walk_pool_walks=cap, walk_spill=True, visit_counts=True, **cfg) as e:
        e.graph_load(g.row_ptr, g.col, P)
        if app == LT.PAGERANK:
            e.walks_init_pagerank(starts, length, param, seed)
        else:
            e.walks_init(starts, app, length if app == LT.DEEPWALK else param, seed)
        e.run()
        paths, lengths = e.get_paths()
        counts = e.visit_counts()
        ps = e.pool_state()
        st = e.stats()
    op, ol, osteps, _ = oracle_for(g, starts, app, param, seed, length)
    np.testing.assert_array_equal(lengths, ol)
    np.testing.assert_array_equal(paths, op)
    np.testing.assert_array_equal(counts, O.visit_counts(op, ol, g.n))
    assert st["steps"] == osteps
    assert ps["device_err"] == 0 and ps["pending"] == 0 and ps["host_chunks"] == 0
    assert ps["free_chunks"] + ps["ring_chunks"] == ps["total_chunks"]
    return st


@pytest.mark.parametrize("cap_div", [3, 8])
@pytest.mark.parametrize("P", [4, 16, 64])
@pytest.mark.parametrize("refill", [0, 2])
def test_spill_deepwalk_exact(gpu, g14, cap_div, P, refill):
    W = 4 * g14.n
    C = 256
    st = run_spill(g14, lt_inputs.deepwalk_starts(W, g14.n), LT.DEEPWALK, 0, 3, P, W // cap_div, chunk_walks=C,
                   refill=refill)
    assert st["spilled_chunks"] > 0
    assert st["reloaded_chunks"] == st["spilled_chunks"]  # every evicted chunk came back
    assert st["spill_d2h_bytes"] == st["spilled_chunks"] * C * 16 == st["spill_h2d_bytes"]
    assert st["chunks_total"] <= 2 * -(-(W // cap_div) // C) + 2 * P + 64  # sized by the cap, not by W
    assert st["host_chunks_peak"] > 0
    assert st["spill_prefetched_chunks"] <= st["reloaded_chunks"]


@pytest.mark.parametrize("app,param", [(LT.PPR, 0.15), (LT.PAGERANK, 0.2)])
@pytest.mark.parametrize("policy", [LT.POLICY_SELECTIVE, LT.POLICY_ROUND_ROBIN])
def test_spill_apps_and_policies(gpu, g14, app, param, policy):
    W = 3 * g14.n
    starts = lt_inputs.ppr_starts(W, g14.argmax_deg) if app == LT.PPR else lt_inputs.deepwalk_starts(W, g14.n)
    st = run_spill(g14, starts, app, param, 5, 8, W // 5, chunk_walks=512, policy=policy)
    assert st["spilled_chunks"] > 0


@pytest.mark.parametrize("C", [64, 1024])
def test_spill_chunk_sizes_and_tiny_pool(gpu, g14, C):
    """A pool only a few chunks larger than the per-launch append reserve: launches are cut at the free
    chunks (tail_cap) and a partition is consumed over several launches."""
    W = 2 * g14.n
    run_spill(g14, lt_inputs.deepwalk_starts(W, g14.n), LT.DEEPWALK, 0, 7, 4, 4 * C, length=9, chunk_walks=C)


@pytest.mark.parametrize("zero_copy,cont", [(False, False), (True, True)])
def test_spill_out_of_core(gpu, g14, zero_copy, cont):
    """Walk spill together with the out-of-core graph pool (the paper's setting: neither the graph nor
    the walks fit the GPU), with zero copy and continuation into resident partitions."""
    P = 16
    b = LT.partition_bounds(g14.row_ptr, P).astype(np.int64)
    rp = g14.row_ptr.astype(np.int64)
    blk = ((max(8 * (b[k + 1] - b[k] + 1) for k in range(P)) + 255) // 256 * 256 +
           max(4 * (rp[b[k + 1]] - rp[b[k]]) for k in range(P)) + 255) // 256 * 256
    W = 4 * g14.n
    st = run_spill(g14, lt_inputs.deepwalk_starts(W, g14.n), LT.DEEPWALK, 0, 2, P, W // 6, chunk_walks=256,
                   graph_pool_bytes=4 * blk, zero_copy=zero_copy, continue_resident=cont)
    assert st["out_of_core"] == 1 and st["spilled_chunks"] > 0


def test_spill_repeated_epochs(gpu, g14):
    """Two epochs on one engine: the host store and staging are reused, statistics are per epoch."""
    W = 3 * g14.n
    starts = lt_inputs.deepwalk_starts(W, g14.n)
    with LT.Engine(walk_pool_walks=W // 4, walk_spill=True, chunk_walks=256) as e:
        e.graph_load(g14.row_ptr, g14.col, 8)
        for seed in (1, 2):
            e.walks_init(starts, LT.DEEPWALK, 12, seed)
            e.run()
            paths, lengths = e.get_paths()
            op, ol, _, _ = O.walks(g14.row_ptr, g14.col, starts, app=O.DEEPWALK, length=12, seed=seed)
            np.testing.assert_array_equal(paths, op)
            st = e.stats()
            assert st["reloaded_chunks"] == st["spilled_chunks"] > 0
