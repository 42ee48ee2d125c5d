"""Parity with CSR offsets at and above 2^32 (Table II :277-285: edge counts in the billions,
so row_ptr is u64). Every other GPU test has m < 2^32, where the high word of an offset is always 0:
this module builds an FS-shaped R-MAT graph at scale 26 with 2.4·10^9 tuples (m ≈ 4.6·10^9 CSR
entries > 2^32) and checks the kernels that carry or rebase offsets, bit-exact against the oracle on
>= 1M sampled walks (the walk definition):

  * the CSR step (row_ptr pair + col gather), the 16-B ADJ entry's .w word, ADJ12's 40-bit packing;
  * the partitioned path (records, findPartition, insertion) at P = 16;
  * out of core at P = 64 (graph-pool block slices whose first edge is past 2^32, continuation into
    resident partitions, next-load prefetch, adaptive zero copy from the mapped host CSR);
  * range ownership at R = 2 over owned ADJ slices (rank 1's slice rebased by ebase ≈ m/2).

Each test also asserts that the sampled oracle paths really step through vertices whose offset is
>= 2^32, so the high word is exercised, not just present."""
import threading

import numpy as np
import pytest

import lt_inputs
import oracle as O
import paper_conf_icde_xing0wxl23_b200 as LT
from paper_conf_icde_xing0wxl23_b200 import dist as ltdist

pytestmark = pytest.mark.gpu

SCALE, TUPLES = 26, 2_400_000_000
L = 80
SAMPLE = 1_000_000


def sample_ids(W, k=SAMPLE, seed=0):
    """The first and last 1000 walks plus a uniform sample (walk w starts at vertex w mod n, so the
    last walks start at the highest-offset vertices)."""
    rng = np.random.default_rng(seed)
    idx = np.unique(np.concatenate([np.arange(min(W, 1000)), np.arange(max(0, W - 1000), W),
                                    rng.integers(0, W, size=k)]))
    return idx.astype(np.uint64)


@pytest.fixture(scope="module")
def big(gpu):
    import torch
    g = lt_inputs.rmat_gpu(SCALE, TUPLES, seed=1)
    assert g.m > (1 << 32) + (1 << 28), g.m
    host = lt_inputs.Graph(g.n, g.m, g.row_ptr.cpu().numpy().view(np.uint64), g.col.cpu().numpy().view(np.uint32),
                           g.max_deg, g.argmax_deg)
    yield g, host
    del g
    torch.cuda.empty_cache()


def high_steps(host, paths, lengths):
    """Path entries (after the start) at vertices whose CSR offset is >= 2^32."""
    hi = host.row_ptr[:-1] >= np.uint64(1 << 32)
    cnt = 0
    for t in range(1, paths.shape[1]):
        live = lengths > t
        cnt += int(np.count_nonzero(hi[paths[live, t]]))
    return cnt


def check_sample(e, host, starts, ids, app=O.DEEPWALK, length=L, alpha=0.15):
    gp, gl = e.get_paths_rows(ids)
    op, ol, _, _ = O.walks(host.row_ptr, host.col, starts[ids.astype(np.int64)], app=app, length=length,
                           alpha=alpha, seed=1, ids=ids)
    np.testing.assert_array_equal(gl, ol)
    np.testing.assert_array_equal(gp, op)
    hs = high_steps(host, op, ol)
    assert hs > 0.01 * len(ids), f"only {hs} sampled steps at offsets >= 2^32"
    return hs


@pytest.mark.parametrize("layout", [LT.LAYOUT_ADJ, LT.LAYOUT_ADJ12, LT.LAYOUT_CSR])
def test_big_offsets_one_partition(big, layout):
    """The bench's launch configuration (P = 1, lane refill, direct start) in each layout."""
    import torch
    g, host = big
    W = g.n
    starts = lt_inputs.deepwalk_starts(W, g.n)
    with LT.Engine(layout=layout) as e:
        e.graph_load(g.row_ptr, g.col, 1)
        assert e.stats()["layout"] == layout
        e.walks_init(torch.from_numpy(starts.view(np.int32)).cuda(), LT.DEEPWALK, L, 1)
        e.run()
        st = e.stats()
        assert st["steps"] == W * L and st["direct_start"] == 1
        check_sample(e, host, starts, sample_ids(W))


@pytest.mark.parametrize("layout", [LT.LAYOUT_ADJ, LT.LAYOUT_CSR])
def test_big_offsets_partitioned(big, layout):
    """P = 16: walk records, findPartition and insertion carry walks across partitions."""
    import torch
    g, host = big
    W = 8_000_000
    starts = lt_inputs.deepwalk_starts(W, g.n, first_walk_id=g.n - W // 2)  # half of them at the top IDs
    with LT.Engine(layout=layout) as e:
        e.graph_load(g.row_ptr, g.col, 16)
        e.walks_init(torch.from_numpy(starts.view(np.int32)).cuda(), LT.DEEPWALK, L, 1, first_walk_id=0)
        e.run()
        assert e.pool_state()["device_err"] == 0
        assert e.stats()["visits"] > W
        check_sample(e, host, starts, sample_ids(W, k=SAMPLE // 2, seed=1))


def test_big_offsets_ppr_partitioned(big):
    import torch
    g, host = big
    W = 4_000_000
    starts = lt_inputs.ppr_starts(W, g.argmax_deg)
    with LT.Engine(layout=LT.LAYOUT_ADJ) as e:
        e.graph_load(g.row_ptr, g.col, 8)
        e.walks_init(torch.from_numpy(starts.view(np.int32)).cuda(), LT.PPR, 0.15, 1)
        e.run()
        ids = sample_ids(W, k=SAMPLE // 2, seed=2)
        gp, gl = e.get_paths_rows(ids)
    op, ol, _, _ = O.walks(host.row_ptr, host.col, starts[ids.astype(np.int64)], app=O.PPR, alpha=0.15, seed=1,
                           ids=ids)
    np.testing.assert_array_equal(gl, ol)
    np.testing.assert_array_equal(gp, op)
    assert high_steps(host, op, ol) > 1000


@pytest.mark.parametrize("prefetch,zero_copy", [(True, True), (True, False), (False, False)])
def test_big_offsets_out_of_core(big, prefetch, zero_copy):
    """Out of core at P = 64 with a 6 GiB graph pool: partition slices past 2^32 are copied into
    graph-pool blocks (rebased by their first edge), walks continue into resident blocks, small buckets
    are served from the mapped host CSR (zero copy)."""
    g, host = big
    W = 3_000_000
    first = g.n - W // 3
    starts = lt_inputs.deepwalk_starts(W, g.n, first_walk_id=first)
    with LT.Engine(graph_pool_bytes=6 << 30, zero_copy=zero_copy, continue_resident=True,
                   ooc_prefetch=prefetch) as e:
        e.graph_load(g.row_ptr, g.col, 64)  # the device CSR is copied into pinned host memory (G_cpu)
        e.walks_init(starts, LT.DEEPWALK, L, 1)
        e.run()
        st = e.stats()
        assert st["out_of_core"] == 1 and st["steps"] == W * L
        if zero_copy:  # ~47K walks per partition: alpha * w < S_p, every launch reads the mapped host CSR
            assert st["zero_copy_launches"] > 0
        else:
            assert st["explicit_copies"] > 0
        check_sample(e, host, starts, sample_ids(W, k=SAMPLE // 2, seed=3))


def test_big_offsets_ownership_adj_slices(big):
    """Range ownership at R = 2 (threaded ranks on one GPU): each rank builds the ADJ entries of its owned
    slice only; rank 1's slice starts near m/2 and its offsets run past 2^32."""
    import torch
    g, host = big
    world, W = 2, 2_000_000
    starts = lt_inputs.deepwalk_starts(W, g.n, first_walk_id=g.n - W // 2)
    ids = sample_ids(W, k=SAMPLE // 2, seed=4)
    hub = ltdist.ThreadComm.Hub(world)
    out, errors = [None] * world, []

    def rank_main(r):
        try:
            with LT.Engine(rank=r, world=world, layout=LT.LAYOUT_ADJ) as e:
                e.graph_load(g.row_ptr, g.col, world)
                e.walks_init(starts, LT.DEEPWALK, L, 1)
                comm = ltdist.ThreadComm(hub, r)
                ltdist.attach_peers(e, comm, W)
                cnt = ltdist.run_supersteps_p2p_fused(e, comm, "cuda")
                paths, lengths = ltdist.merge_paths(e, comm)
                sel = torch.from_numpy(ids.astype(np.int64)).cuda()
                out[r] = (paths[sel].cpu().numpy().view(np.uint32), lengths[sel].cpu().numpy().view(np.uint32),
                          cnt, e.stats())
                del paths, lengths
                torch.cuda.synchronize()
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
    op, ol, _, _ = O.walks(host.row_ptr, host.col, starts[ids.astype(np.int64)], app=O.DEEPWALK, length=L, seed=1,
                           ids=ids)
    for gp, gl, cnt, st in out:
        np.testing.assert_array_equal(gl, ol)
        np.testing.assert_array_equal(gp, op)
    assert sum(o[3]["steps"] for o in out) == W * L
    assert out[1][3]["graph_device_bytes"] > 0
    assert high_steps(host, op, ol) > 0.01 * len(ids)
