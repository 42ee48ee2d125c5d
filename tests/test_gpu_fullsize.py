"""Full-size parity: BASELINE.json configs[3] (FS-shaped, the bench workload) and configs[2]
(TW-shaped PPR) at their full sizes, in the launch configuration bench.py times (library defaults,
P = 1, layout auto). The oracle recomputes a spread sample of >= 1M walks one by one (plus, for PPR,
every walk of length >= 40: the tail of the geometric law); properties that hold at any
size are checked on every walk."""
import numpy as np
import pytest

import lt_inputs
import oracle as O
import paper_conf_icde_xing0wxl23_b200 as LT

pytestmark = pytest.mark.gpu


def _host(g):
    return lt_inputs.Graph(g.n, g.m, g.row_ptr.cpu().numpy().view(np.uint64), g.col.cpu().numpy().view(np.uint32),
                           g.max_deg, g.argmax_deg)


def _sample(W, k=1_000_000, seed=0):
    rng = np.random.default_rng(seed)
    idx = np.unique(np.concatenate([np.arange(min(W, 1000)), np.arange(max(0, W - 1000), W),
                                    rng.integers(0, W, size=k)]))
    return idx.astype(np.uint64)


@pytest.fixture(scope="module")
def fs_graph(gpu):
    c = lt_inputs.CONFIGS[4]
    return lt_inputs.rmat_gpu(c["scale"], c["tuples"], seed=1)


def test_cfg4_fs_shaped_deepwalk_full_size(fs_graph):
    import torch
    g = fs_graph
    W = g.n
    starts = lt_inputs.deepwalk_starts(W, g.n)
    with LT.Engine() as e:
        e.graph_load(g.row_ptr, g.col, 1)
        e.walks_init(torch.from_numpy(starts.view(np.int32)).cuda(), LT.DEEPWALK, 80, 1)
        e.run()
        st = e.stats()
        assert st["layout"] == LT.LAYOUT_ADJ
        assert st["steps"] == W * 80                     # every walk has l steps (no dead ends)
        ids = _sample(W)
        gp, gl = e.get_paths_rows(ids)
        _, lengths = e.get_paths(paths=False)
    assert np.all(lengths == 81)
    gh = _host(g)
    ii = ids.astype(np.int64)
    op, ol, _, _ = O.walks(gh.row_ptr, gh.col, starts[ii], app=O.DEEPWALK, length=80, seed=1, ids=ids)
    np.testing.assert_array_equal(gl, ol)
    np.testing.assert_array_equal(gp, op)


def test_cfg4_partitioned_csr_sampled(fs_graph):
    """The partitioned path (P=16, CSR layout) at full size, same sample."""
    import torch
    g = fs_graph
    W = g.n
    starts = lt_inputs.deepwalk_starts(W, g.n)
    ids = _sample(W, k=1_000_000, seed=3)
    with LT.Engine(layout=LT.LAYOUT_CSR) as e:
        e.graph_load(g.row_ptr, g.col, 16)
        e.walks_init(torch.from_numpy(starts.view(np.int32)).cuda(), LT.DEEPWALK, 80, 1)
        e.run()
        gp, gl = e.get_paths_rows(ids)
        assert e.pool_state()["device_err"] == 0
    gh = _host(g)
    op, ol, _, _ = O.walks(gh.row_ptr, gh.col, starts[ids.astype(np.int64)], app=O.DEEPWALK, length=80, seed=1,
                           ids=ids)
    np.testing.assert_array_equal(gp, op)


def test_cfg3_tw_shaped_ppr_full_size(gpu):
    import torch
    c = lt_inputs.CONFIGS[3]
    g = lt_inputs.rmat_gpu(c["scale"], c["tuples"], seed=1)
    W = g.n
    starts = lt_inputs.ppr_starts(W, g.argmax_deg)
    with LT.Engine() as e:
        e.graph_load(g.row_ptr, g.col, 1)
        e.walks_init(torch.from_numpy(starts.view(np.int32)).cuda(), LT.PPR, 0.15, 1)
        e.run()
        st = e.stats()
        _, lengths = e.get_paths(paths=False)
        # a spread sample plus the whole tail: every walk with >= 40 path vertices (about 0.85^39 of W)
        tail = np.nonzero(lengths >= 40)[0].astype(np.uint64)
        assert len(tail) > 10_000
        ids = np.union1d(_sample(W), tail).astype(np.uint64)
        gp, gl = e.get_paths_rows(ids)
    # geometric length law at full size: mean within 4 sigma of 1/alpha
    N = lengths.astype(np.float64)
    assert abs(N.mean() - 1 / 0.15) < 4 * np.sqrt(0.85 / 0.15 ** 2 / W)
    assert st["steps"] == int((lengths.astype(np.int64) - 1).sum())
    gh = _host(g)
    ii = ids.astype(np.int64)
    op, ol, _, otr = O.walks(gh.row_ptr, gh.col, starts[ii], app=O.PPR, alpha=0.15, seed=1, ids=ids)
    np.testing.assert_array_equal(gl, ol)
    np.testing.assert_array_equal(gp, op)
