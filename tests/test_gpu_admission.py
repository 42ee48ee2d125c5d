"""massive walk counts with a capped walk pool ("walk pool"; the paper's
multi-round comparison, :353-363). With lt_config.walk_pool_walks = m_w < W the walks are admitted in
index order as the pool drains, so at most m_w walks are ever live. Paths, lengths and visit counts must
equal the oracle bit-exactly whatever the cap, partition count, residency mode and application."""
import numpy as np
import pytest

import lt_inputs
import oracle as O
import paper_conf_icde_xing0wxl23_b200 as LT

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def cfg1():
    return lt_inputs.rmat_cpu(12, 65_536, seed=1)


def oracle_for(g, starts, app, param, seed, length=12):
    if app == LT.DEEPWALK:
        return O.walks(g.row_ptr, g.col, starts, app=O.DEEPWALK, length=int(param), seed=seed)
    if app == LT.PPR:
        return O.walks(g.row_ptr, g.col, starts, app=O.PPR, alpha=param, seed=seed)
    return O.walks(g.row_ptr, g.col, starts, app=O.PAGERANK, length=length, alpha=param, seed=seed)


def init(e, starts, app, param, seed, length=12):
    if app == LT.PAGERANK:
        e.walks_init_pagerank(starts, length, param, seed)
    else:
        e.walks_init(starts, app, param, seed)


@pytest.mark.parametrize("cap", [64, 1000, 7000])
@pytest.mark.parametrize("P", [1, 4])
@pytest.mark.parametrize("app,param", [(LT.DEEPWALK, 15), (LT.PPR, 0.15), (LT.PAGERANK, 0.2)])
def test_admission_exact(gpu, cfg1, cap, P, app, param):
    W = 20_000
    starts = lt_inputs.ppr_starts(W, cfg1.argmax_deg) if app == LT.PPR else lt_inputs.deepwalk_starts(W, cfg1.n)
    with LT.Engine(walk_pool_walks=cap, chunk_walks=64, visit_counts=True) as e:
        e.graph_load(cfg1.row_ptr, cfg1.col, P)
        init(e, starts, app, param, 4)
        e.run()
        paths, lengths = e.get_paths()
        counts = e.visit_counts()
        st = e.stats()
    op, ol, osteps, _ = oracle_for(cfg1, starts, app, param, 4)
    np.testing.assert_array_equal(lengths, ol)
    np.testing.assert_array_equal(paths, op)
    np.testing.assert_array_equal(counts, O.visit_counts(op, ol, cfg1.n))
    assert st["steps"] == osteps
    assert st["admissions"] >= -(-W // cap) and st["peak_live"] <= cap
    assert st["chunks_total"] <= 2 * -(-cap // 64) + 2 * P + 64  # the pool is sized by the cap, not by W


def test_admission_out_of_core_with_continuation(gpu):
    g = lt_inputs.rmat_cpu(14, 16 * 2 ** 14, seed=2)
    P = 16
    b = LT.partition_bounds(g.row_ptr, P).astype(np.int64)
    rp = g.row_ptr.astype(np.int64)
    block = ((max(8 * (b[k + 1] - b[k] + 1) for k in range(P)) + 255) // 256 * 256
             + max(4 * (rp[b[k + 1]] - rp[b[k]]) for k in range(P)) + 255) // 256 * 256
    starts = lt_inputs.deepwalk_starts(3 * g.n, g.n)
    with LT.Engine(walk_pool_walks=g.n // 2, graph_pool_bytes=3 * block, zero_copy=True,
                   continue_resident=True) as e:
        e.graph_load(g.row_ptr, g.col, P)
        e.walks_init(starts, LT.DEEPWALK, 10, 6)
        e.run()
        paths, lengths = e.get_paths()
        st = e.stats()
    op, ol, _, _ = O.walks(g.row_ptr, g.col, starts, app=O.DEEPWALK, length=10, seed=6)
    np.testing.assert_array_equal(paths, op)
    assert st["admissions"] > 1 and st["out_of_core"] == 1


def test_paths_off_with_counts_and_admission(gpu, cfg1):
    """path_mode 2 (no path matrix: the paper's accounting for PageRank / PPR) with visit
    counts and a capped pool: lengths and counts still exact; path copy-outs are refused."""
    W = 50_000
    starts = lt_inputs.deepwalk_starts(W, cfg1.n)
    with LT.Engine(path_mode=2, visit_counts=True, walk_pool_walks=4096) as e:
        e.graph_load(cfg1.row_ptr, cfg1.col, 2)
        e.walks_init_pagerank(starts, 10, 0.15, 9)
        e.run()
        _, lengths = e.get_paths(paths=False)
        counts = e.visit_counts()
        with pytest.raises(LT.LTError):
            e.get_paths()
        with pytest.raises(LT.LTError):
            e.get_paths_compact()
    op, ol, _, _ = O.walks(cfg1.row_ptr, cfg1.col, starts, app=O.PAGERANK, length=10, alpha=0.15, seed=9)
    np.testing.assert_array_equal(lengths, ol)
    np.testing.assert_array_equal(counts, O.visit_counts(op, ol, cfg1.n))


def test_long_pagerank_converges(gpu, cfg1):
    """PageRank longer than L_max (the scheduler's sweep bound uses the walk length, not L_max)."""
    starts = lt_inputs.deepwalk_starts(500, cfg1.n)
    with LT.Engine() as e:
        e.graph_load(cfg1.row_ptr, cfg1.col, 8)
        e.walks_init_pagerank(starts, 300, 0.1, 2)
        e.run()
        paths, lengths = e.get_paths()
    op, ol, _, _ = O.walks(cfg1.row_ptr, cfg1.col, starts, app=O.PAGERANK, length=300, alpha=0.1, seed=2)
    np.testing.assert_array_equal(paths, op)


def test_admission_rejected_with_ranks(gpu, cfg1):
    with LT.Engine(walk_pool_walks=100, rank=0, world=2) as e:
        e.graph_load(cfg1.row_ptr, cfg1.col, 4)
        with pytest.raises(LT.LTError) as ei:
            e.walks_init(lt_inputs.deepwalk_starts(1000, cfg1.n), LT.DEEPWALK, 5, 1)
        assert ei.value.status == 1
