"""BASELINE.json configs[4] (UK-shaped Kronecker scale 28, 5.5·10^9 tuples: 129.2M vertices, 10.82·10^9 CSR
entries, offsets up to 2^33.3) on one B200, bit-exact against the oracle on >= 1M sampled walks:

  * the CSR layout with |V| walks, as bench.py runs it on one GPU (layout auto keeps CSR: the augmented
    arrays lie past the 64 GiB gather reach);
  * the compact 12-B augmented layout (ADJ12, 130 GB: 40-bit offsets whose high byte is non-zero);
  * the partitioned path at P = 32 (Kronecker relabelling scatters hubs over every partition).
The graph is built on the GPU by the ranged generator (lt_inputs.rmat_gpu falls back to it when the
one-shot key arrays do not fit)."""
import numpy as np
import pytest

import lt_inputs
import oracle as O
import paper_conf_icde_xing0wxl23_b200 as LT

pytestmark = pytest.mark.gpu
L = 80


def sample_ids(W, k=1_000_000, seed=0):
    rng = np.random.default_rng(seed)
    idx = np.unique(np.concatenate([np.arange(min(W, 1000)), np.arange(max(0, W - 1000), W),
                                    rng.integers(0, W, size=k)]))
    return idx.astype(np.uint64)


@pytest.fixture(scope="module")
def cfg5(gpu):
    import torch
    torch.cuda.empty_cache()
    c = lt_inputs.CONFIGS[5]
    g = lt_inputs.rmat_gpu(c["scale"], c["tuples"], seed=1, permute=c["permute"])
    assert g.m > (1 << 33), g.m
    host = lt_inputs.Graph(g.n, g.m, g.row_ptr.cpu().numpy().view(np.uint64), g.col.cpu().numpy().view(np.uint32),
                           g.max_deg, g.argmax_deg)
    yield g, host
    del g
    torch.cuda.empty_cache()


def check(e, host, starts, ids):
    gp, gl = e.get_paths_rows(ids)
    op, ol, _, _ = O.walks(host.row_ptr, host.col, starts[ids.astype(np.int64)], app=O.DEEPWALK, length=L, seed=1,
                           ids=ids)
    np.testing.assert_array_equal(gl, ol)
    np.testing.assert_array_equal(gp, op)
    hi = host.row_ptr[:-1] >= np.uint64(1 << 33)  # offsets with the 2^33 bit set
    assert int(np.count_nonzero(hi[op[:, 1:]])) > 0.01 * len(ids)


def test_cfg5_csr_full_walks(cfg5):
    import torch
    g, host = cfg5
    W = g.n
    starts = lt_inputs.deepwalk_starts(W, g.n)
    with LT.Engine() as e:
        e.graph_load(g.row_ptr, g.col, 1)
        assert e.stats()["layout"] == LT.LAYOUT_CSR
        e.walks_init(torch.from_numpy(starts.view(np.int32)).cuda(), LT.DEEPWALK, L, 1)
        e.run()
        assert e.stats()["steps"] == W * L
        check(e, host, starts, sample_ids(W))


def test_cfg5_adj12(cfg5):
    import torch
    g, host = cfg5
    W = 4_000_000
    starts = lt_inputs.deepwalk_starts(W, g.n, first_walk_id=g.n - W // 2)
    with LT.Engine(layout=LT.LAYOUT_ADJ12) as e:
        e.graph_load(g.row_ptr, g.col, 1)
        assert e.stats()["layout"] == LT.LAYOUT_ADJ12
        e.walks_init(torch.from_numpy(starts.view(np.int32)).cuda(), LT.DEEPWALK, L, 1)
        e.run()
        check(e, host, starts, sample_ids(W, k=500_000, seed=1))


def test_cfg5_partitioned_csr(cfg5):
    import torch
    g, host = cfg5
    W = 8_000_000
    starts = lt_inputs.deepwalk_starts(W, g.n, first_walk_id=g.n - W // 2)
    with LT.Engine(layout=LT.LAYOUT_CSR) as e:
        e.graph_load(g.row_ptr, g.col, 32)
        e.walks_init(torch.from_numpy(starts.view(np.int32)).cuda(), LT.DEEPWALK, L, 1)
        e.run()
        assert e.pool_state()["device_err"] == 0
        check(e, host, starts, sample_ids(W, k=500_000, seed=2))
