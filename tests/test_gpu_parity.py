"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, walk by walk, bit-exact.

Paths are integer data, so the bar is exact equality of every path entry and every length
(paths are a pure function of CSR, starts, app, parameter, seed and L_max, and must
not depend on P, chunk size, scheduling policy, insertion mode or launch shape).
"""
import numpy as np
import pytest

import lt_inputs
import oracle as O
import paper_conf_icde_xing0wxl23_b200 as LT

pytestmark = pytest.mark.gpu


def run_gpu(g, starts, app, param, seed, P, first=0, device_inputs=False, **cfg):
    import torch
    with LT.Engine(**cfg) as e:
        if device_inputs:
            rp = torch.from_numpy(g.row_ptr.view(np.int64)).cuda()
            col = torch.from_numpy(g.col.view(np.int32)).cuda()
            st = torch.from_numpy(np.ascontiguousarray(starts).view(np.int32)).cuda()
            e.graph_load(rp, col, P)
            e.walks_init(st, app, param, seed, first)
        else:
            e.graph_load(g.row_ptr, g.col, P)
            e.walks_init(starts, app, param, seed, first)
        e.run()
        # path_mode 2 stores no path matrix: only the lengths can be read back
        paths, lengths = e.get_paths(paths=False if cfg.get("path_mode") == 2 else None)
        return paths, lengths, e.stats(), e.bounds()


def run_oracle(g, starts, app, param, seed, first=0, lmax=O.DEFAULT_LMAX):
    ids = np.arange(first, first + len(starts), dtype=np.uint64)
    kw = dict(app=app, seed=seed, ids=ids, lmax=lmax)
    if app == O.DEEPWALK:
        kw["length"] = int(param)
    else:
        kw["alpha"] = param
    return O.walks(g.row_ptr, g.col, starts, **kw)


def assert_parity(g, starts, app, param, seed, P, first=0, **cfg):
    paths, lengths, st, bounds = run_gpu(g, starts, app, param, seed, P, first=first, **cfg)
    op, ol, osteps, otrunc = run_oracle(g, starts, app, param, seed, first=first,
                                        lmax=cfg.get("ppr_max_len", O.DEFAULT_LMAX))
    np.testing.assert_array_equal(lengths, ol)
    np.testing.assert_array_equal(paths, op)
    assert st["steps"] == osteps
    assert st["truncated"] == otrunc
    assert st["num_walks"] == len(starts)
    if len(starts):
        assert st["visits"] >= len(starts)
        if P == 1:
            assert st["visits"] == len(starts) and st["update_launches"] == 1
    assert len(bounds) == P + 1
    return st


@pytest.fixture(scope="module")
def cfg1():
    """BASELINE.json configs[0]: R-MAT scale 12, 65,536 tuples, 4096 DeepWalk walks, l=10, P=4."""
    return lt_inputs.rmat_cpu(12, 65_536, seed=1)


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_cfg1_deepwalk_exact(gpu, cfg1, seed):
    starts = lt_inputs.deepwalk_starts(4096, cfg1.n)
    st = assert_parity(cfg1, starts, LT.DEEPWALK, 10, seed, P=4)
    assert st["steps"] == 4096 * 10


@pytest.mark.parametrize("P", [1, 2, 3, 7, 64, 1000, 3336])
def test_deepwalk_invariant_to_partition_count(gpu, cfg1, P):
    starts = lt_inputs.deepwalk_starts(4096, cfg1.n)
    assert_parity(cfg1, starts, LT.DEEPWALK, 10, 1, P=min(P, cfg1.n))


@pytest.mark.parametrize("P", [8191, 8192, 12_000, 0])
def test_partition_bounds_beyond_shared_memory(gpu, P):
    """Partition bounds are staged in shared memory for P < 8192 and read from global memory beyond
    (the exit test and findPartition, a4); P = 0 here means one partition per vertex."""
    g = _g15()
    P = P or g.n
    assert g.n > 12_000
    starts = lt_inputs.deepwalk_starts(g.n, g.n)
    st = assert_parity(g, starts, LT.DEEPWALK, 12, 5, P=P, chunk_walks=256)
    assert st["visits"] > g.n  # walks crossed partitions
    assert_parity(g, lt_inputs.ppr_starts(8000, g.argmax_deg), LT.PPR, 0.2, 6, P=P, chunk_walks=256)


_G15 = {}


def _g15():
    if "g" not in _G15:
        _G15["g"] = lt_inputs.rmat_cpu(15, 16 * 32_768, seed=2)
    return _G15["g"]


@pytest.mark.parametrize("chunk", [64, 128, 1024, 8192])
@pytest.mark.parametrize("insert_mode", [LT.INSERT_WARP_AGGREGATED, LT.INSERT_DIRECT])
@pytest.mark.parametrize("policy", [LT.POLICY_SELECTIVE, LT.POLICY_ROUND_ROBIN])
def test_invariant_to_pool_and_policy(gpu, cfg1, chunk, insert_mode, policy):
    starts = lt_inputs.deepwalk_starts(4096, cfg1.n)
    assert_parity(cfg1, starts, LT.DEEPWALK, 10, 2, P=16, chunk_walks=chunk, insert_mode=insert_mode,
                  policy=policy)


@pytest.mark.parametrize("alpha", [0.15, 0.5])
@pytest.mark.parametrize("P", [1, 4, 64])
def test_ppr_exact(gpu, cfg1, alpha, P):
    starts = lt_inputs.ppr_starts(4096, cfg1.argmax_deg)
    assert_parity(cfg1, starts, LT.PPR, alpha, 5, P=P, chunk_walks=256)


def test_ppr_truncation(gpu, cfg1):
    starts = lt_inputs.ppr_starts(3000, cfg1.argmax_deg)
    st = assert_parity(cfg1, starts, LT.PPR, 0.01, 9, P=8, ppr_max_len=10)
    assert st["truncated"] > 2000


@pytest.mark.parametrize("W", [0, 1, 31, 33, 4097])
def test_ragged_walk_counts(gpu, cfg1, W):
    starts = lt_inputs.deepwalk_starts(W, cfg1.n)
    assert_parity(cfg1, starts, LT.DEEPWALK, 7, 4, P=5)


def test_zero_length_and_dead_ends(gpu):
    g = lt_inputs.small_graph([(0, 1), (1, 3), (3, 4)], n=6)   # vertices 2 and 5 isolated (d == 0)
    starts = np.array([0, 2, 5, 4, 1, 2], dtype=np.uint32)
    assert_parity(g, starts, LT.DEEPWALK, 9, 1, P=3)
    assert_parity(g, starts, LT.DEEPWALK, 0, 1, P=2)
    assert_parity(g, starts, LT.PPR, 0.2, 1, P=6)


def test_first_walk_id_offsets_philox_counter(gpu, cfg1):
    starts = lt_inputs.deepwalk_starts(1000, cfg1.n, first_walk_id=123_456_789)
    assert_parity(cfg1, starts, LT.DEEPWALK, 10, 1, P=4, first=123_456_789)
    assert_parity(cfg1, starts, LT.DEEPWALK, 10, 1, P=4, first=(1 << 32) + 5)


def test_device_inputs(gpu, cfg1):
    starts = lt_inputs.deepwalk_starts(4096, cfg1.n)
    a = run_gpu(cfg1, starts, LT.DEEPWALK, 10, 3, P=4, device_inputs=True)
    b = run_gpu(cfg1, starts, LT.DEEPWALK, 10, 3, P=4)
    np.testing.assert_array_equal(a[0], b[0])
    op, ol, _, _ = run_oracle(cfg1, starts, LT.DEEPWALK, 10, 3)
    np.testing.assert_array_equal(a[0], op)


def test_repeated_epochs_and_sampled_rows(gpu, cfg1):
    starts = lt_inputs.deepwalk_starts(4096, cfg1.n)
    with LT.Engine() as e:
        e.graph_load(cfg1.row_ptr, cfg1.col, 8)
        for seed in (1, 2, 1):
            e.walks_init(starts, LT.DEEPWALK, 10, seed)
            e.run()
            p, l = e.get_paths()
            op, ol, _, _ = run_oracle(cfg1, starts, LT.DEEPWALK, 10, seed)
            np.testing.assert_array_equal(p, op)
        rows = np.array([0, 5, 4095, 77], dtype=np.uint64)
        rp, rl = e.get_paths_rows(rows)
        np.testing.assert_array_equal(rp, op[rows.astype(np.int64)])
        np.testing.assert_array_equal(rl, ol[rows.astype(np.int64)])


def test_errors_are_status_codes(gpu, cfg1):
    with LT.Engine() as e:
        with pytest.raises(LT.LTError) as ei:
            e.walks_init(np.zeros(4, np.uint32), LT.DEEPWALK, 5, 1)
        assert ei.value.status == 2                     # STATE: no graph
        e.graph_load(cfg1.row_ptr, cfg1.col, 4)
        with pytest.raises(LT.LTError) as ei:
            e.run()
        assert ei.value.status == 2                     # STATE: no walks
        with pytest.raises(LT.LTError) as ei:
            e.walks_init(np.array([cfg1.n], np.uint32), LT.DEEPWALK, 5, 1)
        assert ei.value.status == 1                     # INVALID start
        for bad in (-1.0, 2.5):
            with pytest.raises(LT.LTError):
                e.walks_init(np.zeros(4, np.uint32), LT.DEEPWALK, bad, 1)
        for bad in (0.0, 1.0):
            with pytest.raises(LT.LTError):
                e.walks_init(np.zeros(4, np.uint32), LT.PPR, bad, 1)
        e.walks_init(np.zeros(4, np.uint32), LT.DEEPWALK, 5, 1)
        e.run()
        with pytest.raises(LT.LTError):
            e.run()
    with LT.Engine() as e:
        bad_rp = cfg1.row_ptr.copy()
        bad_rp[5] = bad_rp[6] + 1
        with pytest.raises(LT.LTError):
            e.graph_load(bad_rp, cfg1.col, 4)
        bad_col = cfg1.col.copy()
        bad_col[10] = cfg1.n
        with pytest.raises(LT.LTError):
            e.graph_load(cfg1.row_ptr, bad_col, 4)
        with pytest.raises(LT.LTError):
            e.graph_load(cfg1.row_ptr, cfg1.col, cfg1.n + 1)


def test_scale16_two_walks_per_vertex(gpu):
    g = lt_inputs.rmat_cpu(16, 16 * 65_536, seed=1)
    starts = lt_inputs.deepwalk_starts(2 * g.n, g.n)
    assert_parity(g, starts, LT.DEEPWALK, 30, 1, P=32)
    assert_parity(g, lt_inputs.ppr_starts(50_000, g.argmax_deg), LT.PPR, 0.15, 2, P=32)


@pytest.mark.parametrize("P", [1, 16])
def test_cfg2_lj_shaped_full_parity(gpu, P):
    """BASELINE.json configs[1]: LJ-shaped R-MAT scale 22, 69M tuples, |V| DeepWalk walks, l=80,
    HBM-resident; every walk compared."""
    g = _cfg2()
    starts = lt_inputs.deepwalk_starts(g.n, g.n)
    st = assert_parity(g, starts, LT.DEEPWALK, 80, 1, P=P)
    assert st["steps"] == g.n * 80


_CFG2 = {}


def _cfg2():
    if "g" not in _CFG2:
        _CFG2["g"] = lt_inputs.rmat_cpu(22, 69_000_000, seed=1)
    return _CFG2["g"]


@pytest.mark.parametrize("P,chunk,refill", [(1, 8192, 0), (4, 64, 0), (16, 256, 0), (64, 64, 0), (16, 256, 2),
                                            (4, 1024, 2), (64, 512, 2)])
def test_pool_invariants(gpu, cfg1, P, chunk, refill):
    """Conservation of walks and chunks (a6): after init every walk is pending in some bucket and
    every chunk is either free or installed; after the run nothing is pending and nothing leaked."""
    starts = lt_inputs.deepwalk_starts(4096, cfg1.n)
    with LT.Engine(chunk_walks=chunk, refill=refill) as e:
        e.graph_load(cfg1.row_ptr, cfg1.col, P)
        e.walks_init(starts, LT.DEEPWALK, 10, 1)
        s0 = e.pool_state()
        assert s0["device_err"] == 0, s0
        assert s0["pending"] == 4096, s0
        assert s0["free_chunks"] + s0["ring_chunks"] == s0["total_chunks"], s0
        e.run()
        s1 = e.pool_state()
        assert s1["device_err"] == 0 and s1["pending"] == 0, s1
        # only partially consumed chunks (at most one per partition) may stay installed
        assert s1["ring_chunks"] <= P, s1
        assert s1["free_chunks"] + s1["ring_chunks"] == s1["total_chunks"], s1


@pytest.mark.parametrize("layout", [LT.LAYOUT_CSR, LT.LAYOUT_ADJ, LT.LAYOUT_ADJ12])
@pytest.mark.parametrize("ilp,refill", [(1, 1), (2, 1), (4, 1), (1, 2)])
@pytest.mark.parametrize("gather_mode", [0, 3])
@pytest.mark.parametrize("P", [1, 8])
def test_kernel_variants_exact(gpu, cfg1, layout, ilp, refill, gather_mode, P):
    """Layout (CSR vs augmented adjacency), walks per lane, lane refill and cache hints change only
    how the gathers are issued, never which neighbour is chosen."""
    kw = dict(layout=layout, ilp=ilp, gather_mode=gather_mode, chunk_walks=256, refill=refill)
    assert_parity(cfg1, lt_inputs.deepwalk_starts(3000, cfg1.n), LT.DEEPWALK, 12, 7, P=P, **kw)
    assert_parity(cfg1, lt_inputs.ppr_starts(3000, cfg1.argmax_deg), LT.PPR, 0.2, 7, P=P, **kw)
    g = lt_inputs.small_graph([(0, 1), (1, 3), (3, 4)], n=6)
    assert_parity(g, np.array([0, 2, 5, 4, 1, 2], dtype=np.uint32), LT.DEEPWALK, 9, 1, P=min(P, 6), **kw)


def test_layouts_memory_and_limits(gpu, cfg1):
    """Graph bytes per layout (col is released once an augmented layout is built from a host graph; a
    borrowed device col is no longer referenced), and ADJ12's 24-bit degree limit."""
    import torch
    n, m = cfg1.n, cfg1.m
    expect = {LT.LAYOUT_CSR: (n + 1) * 8 + 4 * m, LT.LAYOUT_ADJ: (n + 1) * 8 + 16 * m,
              LT.LAYOUT_ADJ12: (n + 1) * 8 + 12 * m}
    for lay, b in expect.items():
        with LT.Engine(layout=lay) as e:
            e.graph_load(cfg1.row_ptr, cfg1.col, 2)
            st = e.stats()
            assert st["layout"] == lay and st["graph_device_bytes"] == b, (lay, st["graph_device_bytes"], b)
            # borrowed device graph: col is kept referenced only for CSR
            rp = torch.from_numpy(cfg1.row_ptr.view(np.int64)).cuda()
            col = torch.from_numpy(cfg1.col.view(np.int32)).cuda()
            e.graph_load(rp, col, 2)
            assert len(e._graph_keep) == (2 if lay == LT.LAYOUT_CSR else 1)
            del col
            torch.cuda.empty_cache()
            starts = lt_inputs.deepwalk_starts(3000, n)
            e.walks_init(starts, LT.DEEPWALK, 9, 4)
            e.run()
            p_, l_ = e.get_paths()
        op, ol, _, _ = run_oracle(cfg1, starts, LT.DEEPWALK, 9, 4)
        np.testing.assert_array_equal(p_, op)
    # a star whose hub has 2^24 neighbours: too wide for ADJ12's 24-bit degree field
    leaves = 1 << 24
    src = np.concatenate([np.zeros(leaves, np.uint32), np.arange(1, leaves + 1, dtype=np.uint32)])
    row_ptr = np.concatenate([[0, leaves], leaves + np.arange(1, leaves + 1)]).astype(np.uint64)
    col = np.concatenate([np.arange(1, leaves + 1, dtype=np.uint32), np.zeros(leaves, np.uint32)])
    assert len(src) == len(col) == row_ptr[-1]
    with LT.Engine(layout=LT.LAYOUT_ADJ12) as e:
        with pytest.raises(LT.LTError, match="2\\^24"):
            e.graph_load(row_ptr, col, 1)
    with LT.Engine() as e:  # auto falls back to a layout that holds it
        e.graph_load(row_ptr, col, 1)
        assert e.stats()["layout"] in (LT.LAYOUT_ADJ, LT.LAYOUT_CSR)
        e.walks_init(np.array([0, 5, 1 << 24], np.uint32), LT.DEEPWALK, 6, 1)
        e.run()
        p_, l_ = e.get_paths()
    op, ol, _, _ = O.walks(row_ptr, col, np.array([0, 5, 1 << 24], np.uint32), app=O.DEEPWALK, length=6, seed=1)
    np.testing.assert_array_equal(p_, op)


@pytest.mark.parametrize("path_mode", [0, 1])
@pytest.mark.parametrize("P", [1, 3, 16])
@pytest.mark.parametrize("length", [0, 1, 7, 8, 9, 15, 16, 17, 80])
@pytest.mark.parametrize("refill", [1, 2])
def test_path_store_modes_and_sector_edges(gpu, cfg1, path_mode, P, length, refill):
    """Buffered full-sector path stores vs one store per step, at lengths around the 8-entry sector
    boundaries, with visits that start mid-sector (P > 1), with and without lane refill."""
    assert_parity(cfg1, lt_inputs.deepwalk_starts(1500, cfg1.n), LT.DEEPWALK, length, 3, P=P, path_mode=path_mode,
                  refill=refill)


def test_path_mode_off_keeps_lengths(gpu, cfg1):
    starts = lt_inputs.deepwalk_starts(2000, cfg1.n)
    paths, lengths, st, _ = run_gpu(cfg1, starts, LT.PPR, 0.15, 4, P=4, path_mode=2)
    _, ol, osteps, _ = run_oracle(cfg1, starts, LT.PPR, 0.15, 4)
    np.testing.assert_array_equal(lengths, ol)
    assert st["steps"] == osteps


@pytest.mark.parametrize("direct", [True, False])
@pytest.mark.parametrize("path_mode", [0, 1])
@pytest.mark.parametrize("device_inputs", [False, True])
def test_direct_start(gpu, cfg1, direct, path_mode, device_inputs):
    """Direct start (lt_config.direct_start; P == 1): no walk records are written at init, the update
    kernel builds walk j's record from starts[j]. Paths, lengths, steps, visits and the pool invariants
    are those of the record path; the stats say which path ran."""
    W = 5003  # several refill claims of 64 and a ragged tail
    for app, param, starts in ((LT.DEEPWALK, 17, lt_inputs.deepwalk_starts(W, cfg1.n)),
                               (LT.PPR, 0.15, lt_inputs.ppr_starts(W, cfg1.argmax_deg))):
        st = assert_parity(cfg1, starts, app, param, 9, P=1, first=123, path_mode=path_mode,
                           device_inputs=device_inputs, direct_start=direct)
        assert st["direct_start"] == (1 if direct else 0)
        assert st["visits"] == W and st["admissions"] == 1
    # never with several partitions, a walk-pool cap or the per-walk kernel without refill
    st = assert_parity(cfg1, lt_inputs.deepwalk_starts(W, cfg1.n), LT.DEEPWALK, 5, 9, P=2, direct_start=direct)
    assert st["direct_start"] == 0
    st = assert_parity(cfg1, lt_inputs.deepwalk_starts(W, cfg1.n), LT.DEEPWALK, 5, 9, P=1, refill=1,
                       direct_start=direct)
    assert st["direct_start"] == 0
    with LT.Engine(direct_start=direct, chunk_walks=64) as e:
        e.graph_load(cfg1.row_ptr, cfg1.col, 1)
        e.walks_init(lt_inputs.deepwalk_starts(W, cfg1.n), LT.DEEPWALK, 6, 2)
        s0 = e.pool_state()
        assert s0["pending"] == W and s0["device_err"] == 0, s0
        assert s0["free_chunks"] + s0["ring_chunks"] == s0["total_chunks"], s0
        e.run()
        s1 = e.pool_state()
        assert s1["pending"] == 0 and s1["device_err"] == 0, s1
        assert s1["free_chunks"] + s1["ring_chunks"] == s1["total_chunks"], s1
        assert s1["ring_chunks"] == (0 if direct else 1), s1  # direct: no chunk was ever installed
        # a second epoch on the same context (the pool is reset by lt_walks_init)
        e.walks_init(lt_inputs.deepwalk_starts(W, cfg1.n), LT.DEEPWALK, 6, 3)
        e.run()
        _, l2 = e.get_paths(paths=False)
        assert np.all(l2 == 7)


@pytest.mark.parametrize("chunks", [1, 3, 8])
@pytest.mark.parametrize("app,param", [(LT.DEEPWALK, 11), (LT.PPR, 0.2)])
def test_run_to_host_streamed(gpu, cfg1, chunks, app, param):
    import torch
    W = 5000
    starts = lt_inputs.deepwalk_starts(W, cfg1.n) if app == LT.DEEPWALK else lt_inputs.ppr_starts(W, cfg1.argmax_deg)
    S = param + 1 if app == LT.DEEPWALK else O.DEFAULT_LMAX + 1
    paths = torch.empty((W, S), dtype=torch.int32, pin_memory=True)
    lengths = torch.empty(W, dtype=torch.int32, pin_memory=True)
    with LT.Engine() as e:
        e.graph_load(cfg1.row_ptr, cfg1.col, 1)
        e.run_to_host(torch.from_numpy(starts.view(np.int32)), app, param, 6, first_walk_id=17, paths=paths,
                      lengths=lengths, chunks=chunks)
        st = e.stats()
    op, ol, osteps, _ = run_oracle(cfg1, starts, app, param, 6, first=17)
    np.testing.assert_array_equal(lengths.numpy().view(np.uint32), ol)
    np.testing.assert_array_equal(paths.numpy().view(np.uint32), op)
    assert st["steps"] == osteps and st["num_walks"] == W


def _ragged_equals_rows(offsets, vertices, paths, lengths):
    assert offsets[0] == 0 and np.array_equal(np.diff(offsets.astype(np.int64)), lengths.astype(np.int64))
    assert len(vertices) == int(offsets[-1])
    for w in range(len(lengths)):
        np.testing.assert_array_equal(vertices[int(offsets[w]): int(offsets[w + 1])], paths[w, : lengths[w]])


@pytest.mark.parametrize("app,param,W", [(LT.PPR, 0.15, 4096), (LT.PPR, 0.5, 9000), (LT.DEEPWALK, 9, 4097),
                                         (LT.DEEPWALK, 3, 0)])
@pytest.mark.parametrize("P", [1, 4])
def test_compact_paths_equal_oracle(gpu, cfg1, app, param, W, P):
    """lt_get_paths_compact: offsets = exclusive prefix sum of the oracle's lengths, vertices = the
    oracle's rows concatenated (tiles of 4096 lengths: W = 9000 spans a ragged third tile)."""
    starts = (lt_inputs.deepwalk_starts(W, cfg1.n) if app == LT.DEEPWALK else lt_inputs.ppr_starts(W, cfg1.argmax_deg))
    with LT.Engine() as e:
        e.graph_load(cfg1.row_ptr, cfg1.col, P)
        e.walks_init(starts, app, param, 3)
        e.run()
        offsets, vertices = e.get_paths_compact()
        paths, lengths = e.get_paths()  # lazy padding after a compact copy-out
    op, ol, _, _ = run_oracle(cfg1, starts, app, param, 3)
    np.testing.assert_array_equal(paths, op)
    _ragged_equals_rows(offsets, vertices, op, ol)


@pytest.mark.parametrize("chunks", [1, 3])
@pytest.mark.parametrize("app,param", [(LT.PPR, 0.2), (LT.DEEPWALK, 11)])
def test_run_to_host_compact(gpu, cfg1, chunks, app, param):
    W = 10_000
    starts = (lt_inputs.deepwalk_starts(W, cfg1.n) if app == LT.DEEPWALK else lt_inputs.ppr_starts(W, cfg1.argmax_deg))
    with LT.Engine() as e:
        e.graph_load(cfg1.row_ptr, cfg1.col, 1)
        offsets, vertices = e.run_to_host_compact(starts, app, param, 9, 77, chunks=chunks)
        st = e.stats()
    op, ol, osteps, _ = run_oracle(cfg1, starts, app, param, 9, first=77)
    _ragged_equals_rows(offsets, vertices, op, ol)
    assert st["steps"] == osteps


def test_run_to_host_validates_starts_on_device(gpu, cfg1):
    """lt_run_to_host copies every start once and range-checks it on the device: a bad start anywhere
    (here in the last range) fails the call before any walk runs; PageRank is refused (no visit
    counts on this path); the context is usable afterwards."""
    W = 3000
    starts = lt_inputs.deepwalk_starts(W, cfg1.n)
    bad = starts.copy()
    bad[-1] = cfg1.n
    with LT.Engine() as e:
        e.graph_load(cfg1.row_ptr, cfg1.col, 1)
        with pytest.raises(LT.LTError, match="start"):
            e.run_to_host(bad, LT.DEEPWALK, 5, 1, chunks=4)
        with pytest.raises(LT.LTError, match="PageRank"):
            e.run_to_host(starts, LT.PAGERANK, 5, 1, chunks=4)
        paths = np.empty((W, 6), dtype=np.uint32)
        lengths = np.empty(W, dtype=np.uint32)
        e.run_to_host(starts, LT.DEEPWALK, 5, 1, paths=paths, lengths=lengths, chunks=4)
    op, ol, _, _ = run_oracle(cfg1, starts, LT.DEEPWALK, 5, 1)
    np.testing.assert_array_equal(paths, op)
    np.testing.assert_array_equal(lengths, ol)


def test_compact_capacity_error(gpu, cfg1):
    starts = lt_inputs.ppr_starts(2000, cfg1.argmax_deg)
    with LT.Engine() as e:
        e.graph_load(cfg1.row_ptr, cfg1.col, 1)
        with pytest.raises(LT.LTError) as ei:
            e.run_to_host_compact(starts, LT.PPR, 0.15, 1, vertices=np.empty(10, dtype=np.uint32))
        assert ei.value.status == LT.lt.LT_ERR_INVALID


@pytest.mark.parametrize("layout", [LT.LAYOUT_CSR, LT.LAYOUT_ADJ])
def test_lemire_rejection_chain_at_degree_2_31_plus_1(gpu, layout):
    """Reading R4 at its extreme: a vertex of degree d = 2^31 + 1 rejects each word with probability
    (2^32 mod d) / 2^32 ~ 1/2, so the GPU's slow path walks the step's word stream well into Philox
    blocks j >= 1 (1/16 of the draws need a fifth word). Multi-edges make the graph: hub 0 has
    2^31 + 1 entries, entry i pointing to 1 + (i mod 65,535), and every other vertex one edge back to
    0, so each hub step's index shows in the path (mod 65,535) and must equal the oracle's."""
    d = (1 << 31) + 1
    n = 1 << 16
    col = np.empty(d + n - 1, dtype=np.uint32)
    col[:d] = np.resize(np.arange(1, n, dtype=np.uint32), d)  # entry i -> 1 + (i mod 65,535)
    col[d:] = 0
    row_ptr = np.empty(n + 1, dtype=np.uint64)
    row_ptr[0] = 0
    row_ptr[1:] = d + np.arange(n, dtype=np.uint64)
    g = lt_inputs.Graph(n, len(col), row_ptr, col, d, 0)
    starts = np.zeros(20_000, dtype=np.uint32)
    assert_parity(g, starts, LT.DEEPWALK, 12, 3, P=1, layout=layout)
    assert_parity(g, starts, LT.PPR, 0.1, 4, P=3, layout=layout)


@pytest.mark.parametrize("layout", [LT.LAYOUT_CSR, LT.LAYOUT_ADJ, LT.LAYOUT_ADJ12])
@pytest.mark.parametrize("P", [2, 16, 300])
@pytest.mark.parametrize("chunk", [256, 8192])
@pytest.mark.parametrize("refill", [1, 2])
def test_offset_records_exact(gpu, layout, P, chunk, refill):
    """Walk records that carry the current vertex's offset and degree (O records: written by the update
    kernels for walks entering a local bucket, with the augmented layouts) on a graph large enough for
    every partition to exchange walks many times, partitions from 2 to 300, both P > 1 kernels,
    DeepWalk / PPR / PageRank; paths and visit counts equal the oracle."""
    g = lt_inputs.rmat_cpu(15, 16 * 2 ** 15, seed=4)
    kw = dict(layout=layout, refill=refill, chunk_walks=chunk)
    st = assert_parity(g, lt_inputs.deepwalk_starts(3 * g.n, g.n), LT.DEEPWALK, 23, 5, P=P, **kw)
    assert st["visits"] > 3 * g.n
    assert_parity(g, lt_inputs.ppr_starts(50_000, g.argmax_deg), LT.PPR, 0.1, 6, P=P, **kw)
    with LT.Engine(visit_counts=True, **kw) as e:
        starts = lt_inputs.deepwalk_starts(2 * g.n, g.n)
        e.graph_load(g.row_ptr, g.col, P)
        e.walks_init_pagerank(starts, 19, 0.2, 8)
        e.run()
        paths, lengths = e.get_paths()
        counts = e.visit_counts()
    op, ol, _, _ = O.walks(g.row_ptr, g.col, starts, app=O.PAGERANK, length=19, alpha=0.2, seed=8)
    np.testing.assert_array_equal(paths, op)
    np.testing.assert_array_equal(counts, O.visit_counts(op, ol, g.n))

