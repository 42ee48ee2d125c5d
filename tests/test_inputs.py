"""Input generator checks (lt_inputs): the preprocessing PAPER.md:273 states, determinism, and the
CPU/GPU builds agreeing bit-exactly."""
import numpy as np
import pytest

import lt_inputs


def _check_csr(g, scale):
    rp, col = g.row_ptr.astype(np.int64), g.col
    assert rp[0] == 0 and rp[-1] == g.m == len(col)
    assert 0 < g.n <= 2 ** scale
    deg = np.diff(rp)
    assert deg.min() >= 1                       # zero-degree vertices removed
    assert int(deg.max()) == g.max_deg
    assert int(np.argmax(deg)) == g.argmax_deg  # first (smallest) ID among ties
    assert col.max() < g.n
    src = np.repeat(np.arange(g.n, dtype=np.int64), deg)
    assert not np.any(src == col)               # no self loops
    # each adjacency list strictly ascending -> sorted and duplicate-free
    same = src[1:] == src[:-1]
    assert np.all(col[1:][same] > col[:-1][same])
    # symmetric: the multiset of (u,v) equals the multiset of (v,u)
    fwd = src * g.n + col
    bwd = col.astype(np.int64) * g.n + src
    np.testing.assert_array_equal(np.sort(fwd), np.sort(bwd))


@pytest.mark.parametrize("scale,tuples", [(8, 2048), (12, 65536), (14, 16 * 2 ** 14)])
def test_rmat_csr_is_preprocessed(scale, tuples):
    _check_csr(lt_inputs.rmat_cpu(scale, tuples, seed=1), scale)


def test_rmat_deterministic_and_thread_independent():
    a = lt_inputs.rmat_cpu(13, 100_000, seed=3, threads=1)
    b = lt_inputs.rmat_cpu(13, 100_000, seed=3, threads=8)
    assert a.n == b.n and a.m == b.m
    np.testing.assert_array_equal(a.row_ptr, b.row_ptr)
    np.testing.assert_array_equal(a.col, b.col)
    c = lt_inputs.rmat_cpu(13, 100_000, seed=4)
    assert c.m != a.m or not np.array_equal(c.col, a.col)


def test_rmat_quadrant_frequencies_match_initiator():
    # top-level quadrant of tuple e follows (a,b,c,d) = (.57,.19,.19,.05)
    scale, E = 10, 40_000
    q = np.zeros(4)
    for e in range(E):
        u, v = lt_inputs.tuple_at(scale, 9, False, e)
        q[2 * (u >> (scale - 1)) + (v >> (scale - 1))] += 1
    p = np.array([0.57, 0.19, 0.19, 0.05])
    assert np.all(np.abs(q / E - p) < 4 * np.sqrt(p * (1 - p) / E))


def test_kronecker_permutation_is_isomorphic():
    a = lt_inputs.rmat_cpu(11, 30_000, seed=2, permute=False)
    b = lt_inputs.rmat_cpu(11, 30_000, seed=2, permute=True)
    _check_csr(b, 11)
    assert a.n == b.n and a.m == b.m
    np.testing.assert_array_equal(np.sort(np.diff(a.row_ptr.astype(np.int64))),
                                  np.sort(np.diff(b.row_ptr.astype(np.int64))))
    # the permutation moves hubs away from low IDs
    assert b.argmax_deg != a.argmax_deg or b.max_deg == a.max_deg


def test_small_graph_helper():
    g = lt_inputs.small_graph([(0, 1), (1, 2), (1, 2), (2, 2)])
    assert g.n == 3 and g.m == 4
    assert list(g.row_ptr) == [0, 1, 3, 4] and list(g.col) == [1, 0, 2, 1]


def test_starts():
    assert list(lt_inputs.deepwalk_starts(5, 3)) == [0, 1, 2, 0, 1]
    assert list(lt_inputs.deepwalk_starts(3, 4, first_walk_id=6)) == [2, 3, 0]
    assert list(lt_inputs.ppr_starts(3, 7)) == [7, 7, 7]


@pytest.mark.gpu
@pytest.mark.parametrize("scale,tuples,permute", [(12, 65536, False), (16, 16 * 65536, False), (15, 300_000, True)])
def test_gpu_generator_equals_cpu(gpu, scale, tuples, permute):
    c = lt_inputs.rmat_cpu(scale, tuples, seed=1, permute=permute)
    g = lt_inputs.rmat_gpu(scale, tuples, seed=1, permute=permute)
    assert (g.n, g.m, g.max_deg, g.argmax_deg) == (c.n, c.m, c.max_deg, c.argmax_deg)
    np.testing.assert_array_equal(g.row_ptr.cpu().numpy().view(np.uint64), c.row_ptr)
    np.testing.assert_array_equal(g.col.cpu().numpy().view(np.uint32), c.col)


@pytest.mark.gpu
@pytest.mark.parametrize("scale,tuples,permute,max_pass", [(12, 65536, False, 40_000), (15, 300_000, True, 70_000),
                                                          (16, 16 * 65536, False, 10 ** 9), (14, 200_000, True, 400)])
def test_ranged_gpu_generator_equals_cpu(gpu, scale, tuples, permute, max_pass):
    """The ranged build (one source range per pass; configs[4] at scale 28) produces the same CSR as the
    CPU build, with one pass or many (max_pass keys per pass), R-MAT and Kronecker."""
    c = lt_inputs.rmat_cpu(scale, tuples, seed=1, permute=permute)
    if max_pass == 400:  # smaller than the fullest source bin: refused, not truncated
        with pytest.raises(RuntimeError):
            lt_inputs.rmat_gpu_ranged(scale, tuples, seed=1, permute=permute, max_pass_keys=max_pass)
        return
    g = lt_inputs.rmat_gpu_ranged(scale, tuples, seed=1, permute=permute, max_pass_keys=max_pass)
    assert (g.n, g.m, g.max_deg, g.argmax_deg) == (c.n, c.m, c.max_deg, c.argmax_deg)
    assert (g.passes > 1) == (max_pass < 2 * tuples)
    np.testing.assert_array_equal(g.row_ptr.cpu().numpy().view(np.uint64), c.row_ptr)
    np.testing.assert_array_equal(g.col.cpu().numpy().view(np.uint32), c.col)
