"""Range-ownership mode on the real kernels: `world` engines on one GPU, one thread each, exchanging
walk records through dist.ThreadComm (the same superstep driver the NCCL path uses). Merged paths
must equal the oracle bit-exactly for every rank count (paths are independent of
GPU count)."""
import threading

import numpy as np
import pytest

import lt_inputs
import oracle as O
import paper_conf_icde_xing0wxl23_b200 as LT
from paper_conf_icde_xing0wxl23_b200 import dist as ltdist

pytestmark = pytest.mark.gpu


def run_owned(g, starts, app, param, seed, P, world, **cfg):
    import torch
    hub = ltdist.ThreadComm.Hub(world)
    results, errors = [None] * world, []

    def rank_main(r):
        try:
            with LT.Engine(rank=r, world=world, **cfg) as e:
                e.graph_load(g.row_ptr, g.col, P)
                e.walks_init(starts, app, param, seed)
                comm = ltdist.ThreadComm(hub, r)
                counters = ltdist.run_supersteps(e, comm, "cuda")
                paths, lengths = ltdist.merge_paths(e, comm)
                torch.cuda.synchronize()
                results[r] = (paths.cpu().numpy().view(np.uint32), lengths.cpu().numpy().view(np.uint32),
                              counters, e.stats())
        except Exception as ex:  # surface thread failures
            errors.append(ex)
            hub.barrier.abort()

    th = [threading.Thread(target=rank_main, args=(r,)) for r in range(world)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    if errors:
        raise errors[0]
    return results


def oracle_of(g, starts, app, param, seed):
    kw = dict(app=O.DEEPWALK, length=int(param)) if app == LT.DEEPWALK else dict(app=O.PPR, alpha=param)
    return O.walks(g.row_ptr, g.col, starts, seed=seed, **kw)


@pytest.fixture(scope="module")
def g13():
    return lt_inputs.rmat_cpu(13, 8 * 2 ** 13, seed=3)


@pytest.mark.parametrize("world", [2, 3, 4])
@pytest.mark.parametrize("layout", [LT.LAYOUT_CSR, LT.LAYOUT_ADJ, LT.LAYOUT_ADJ12])
def test_ownership_deepwalk_exact(gpu, g13, world, layout):
    starts = lt_inputs.deepwalk_starts(3 * g13.n, g13.n)
    res = run_owned(g13, starts, LT.DEEPWALK, 16, 2, 12, world, layout=layout, chunk_walks=512)
    op, ol, osteps, _ = oracle_of(g13, starts, LT.DEEPWALK, 16, 2)
    for paths, lengths, counters, st in res:
        np.testing.assert_array_equal(lengths, ol)
        np.testing.assert_array_equal(paths, op)
    assert sum(r[3]["steps"] for r in res) == osteps  # each step is taken on exactly one rank
    assert res[0][2]["records_sent"] > 0
    # slice-only graph: a rank holds row_ptr plus the CSR (and ADJ) entries of the
    # vertices it owns; the slices partition the m entries
    per_entry = {LT.LAYOUT_CSR: 4, LT.LAYOUT_ADJ: 16, LT.LAYOUT_ADJ12: 12}[layout]
    slices = [(st["graph_device_bytes"] - (g13.n + 1) * 8) / per_entry for _, _, _, st in res]
    assert all(x == int(x) and 0 < x < g13.m for x in slices), slices
    assert sum(slices) == g13.m
    assert all(st["layout"] == layout for _, _, _, st in res)


def test_ownership_device_graph_slice(gpu, g13):
    """lt_graph_load_device with ownership: the caller's whole device CSR is borrowed, each rank gathers
    only from (and builds ADJ only for) its owned slice."""
    import torch
    world = 3
    starts = lt_inputs.deepwalk_starts(2 * g13.n, g13.n)
    rp = torch.from_numpy(g13.row_ptr.view(np.int64)).cuda()
    col = torch.from_numpy(g13.col.view(np.int32)).cuda()
    g_dev = type("G", (), {"row_ptr": rp, "col": col})
    res = run_owned(g_dev, starts, LT.DEEPWALK, 9, 8, 9, world, layout=LT.LAYOUT_ADJ, chunk_walks=256)
    op, ol, _, _ = oracle_of(g13, starts, LT.DEEPWALK, 9, 8)
    for paths, lengths, _, st in res:
        np.testing.assert_array_equal(lengths, ol)
        np.testing.assert_array_equal(paths, op)
    assert sum((st["graph_device_bytes"] - (g13.n + 1) * 8) // 16 for _, _, _, st in res) == g13.m


@pytest.mark.parametrize("world", [2, 4])
def test_ownership_ppr_exact(gpu, g13, world):
    starts = lt_inputs.ppr_starts(20_000, g13.argmax_deg)
    res = run_owned(g13, starts, LT.PPR, 0.15, 5, 8, world, chunk_walks=256)
    op, ol, _, _ = oracle_of(g13, starts, LT.PPR, 0.15, 5)
    for paths, lengths, _, _ in res:
        np.testing.assert_array_equal(lengths, ol)
        np.testing.assert_array_equal(paths, op)


@pytest.mark.parametrize("cont", [False, True])
def test_ownership_out_of_core_ranks(gpu, g13, cont):
    """Each rank running its owned range out of core (graph pool of 2 blocks), with and without
    continuation into resident partitions (f4)."""
    starts = lt_inputs.deepwalk_starts(g13.n, g13.n)
    res = run_owned(g13, starts, LT.DEEPWALK, 10, 4, 8, 2, graph_pool_bytes=8 << 20, zero_copy=True,
                    continue_resident=cont)
    op, ol, _, _ = oracle_of(g13, starts, LT.DEEPWALK, 10, 4)
    for paths, lengths, _, st in res:
        np.testing.assert_array_equal(paths, op)
        assert st["out_of_core"] == 1
