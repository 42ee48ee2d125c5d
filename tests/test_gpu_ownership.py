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


# ---- peer exchange (lt_exchange_buffers / attach / sent / take): walks for another rank are
# appended by the update kernels straight into that rank's receive buffer (peer memory)

def run_owned_p2p(g, starts, app, param, seed, P, world, capacity=None, **cfg):
    import torch
    hub = ltdist.ThreadComm.Hub(world)
    results, errors = [None] * world, []

    def rank_main(r):
        try:
            with LT.Engine(rank=r, world=world, **cfg) as e:
                e.graph_load(g.row_ptr, g.col, P)
                if app == LT.PAGERANK:
                    e.walks_init_pagerank(starts, int(param[0]), param[1], seed)
                else:
                    e.walks_init(starts, app, param, seed)
                comm = ltdist.ThreadComm(hub, r)
                ltdist.attach_peers(e, comm, capacity or len(starts))
                counters = ltdist.run_supersteps_p2p(e, comm, "cuda")
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


@pytest.mark.parametrize("world", [2, 3, 4])
@pytest.mark.parametrize("layout", [LT.LAYOUT_CSR, LT.LAYOUT_ADJ])
@pytest.mark.parametrize("app,param", [(LT.DEEPWALK, 16), (LT.PPR, 0.15)])
def test_peer_exchange_exact(gpu, g13, world, layout, app, param):
    starts = (lt_inputs.deepwalk_starts(3 * g13.n, g13.n) if app == LT.DEEPWALK
              else lt_inputs.ppr_starts(20_000, g13.argmax_deg))
    res = run_owned_p2p(g13, starts, app, param, 2, 12, world, layout=layout, chunk_walks=512)
    op, ol, osteps, _ = oracle_of(g13, starts, app, param, 2)
    for paths, lengths, counters, st in res:
        np.testing.assert_array_equal(lengths, ol)
        np.testing.assert_array_equal(paths, op)
    assert sum(r[3]["steps"] for r in res) == osteps
    assert res[0][2]["supersteps"] == res[-1][2]["supersteps"]
    assert sum(r[2]["records_sent"] for r in res) > 0


def test_peer_exchange_out_of_core_and_repeat(gpu, g13):
    """Peer exchange with every rank out of core (continuation on), then a second epoch on the same
    engines: the superstep parities stay aligned across epochs."""
    import torch
    world = 2
    hub = ltdist.ThreadComm.Hub(world)
    starts = lt_inputs.deepwalk_starts(g13.n, g13.n)
    out, errors = [None] * world, []

    def rank_main(r):
        try:
            with LT.Engine(rank=r, world=world, graph_pool_bytes=8 << 20, zero_copy=True,
                           continue_resident=True) as e:
                e.graph_load(g13.row_ptr, g13.col, 8)
                comm = ltdist.ThreadComm(hub, r)
                res = []
                for seed in (4, 5):
                    e.walks_init(starts, LT.DEEPWALK, 10, seed)
                    if seed == 4:
                        ltdist.attach_peers(e, comm, len(starts))
                    ltdist.run_supersteps_p2p(e, comm, "cuda")
                    paths, lengths = ltdist.merge_paths(e, comm)
                    torch.cuda.synchronize()
                    res.append(paths.cpu().numpy().view(np.uint32))
                out[r] = res
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
    for i, seed in enumerate((4, 5)):
        op, _, _, _ = oracle_of(g13, starts, LT.DEEPWALK, 10, seed)
        for r in range(world):
            np.testing.assert_array_equal(out[r][i], op)


def test_peer_exchange_overflow_is_an_error(gpu, g13):
    starts = lt_inputs.deepwalk_starts(g13.n, g13.n)
    with pytest.raises(LT.LTError, match="overflow"):
        run_owned_p2p(g13, starts, LT.DEEPWALK, 10, 1, 12, 2, capacity=16)


def _p2p_proc(rank, world, port, out_q, fused=False):
    import os

    import torch
    import torch.distributed as tdist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    tdist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        g = lt_inputs.rmat_cpu(13, 8 * 2 ** 13, seed=3)
        starts = lt_inputs.deepwalk_starts(2 * g.n, g.n)
        with LT.Engine(rank=rank, world=world) as e:
            e.graph_load(g.row_ptr, g.col, world if fused else 2 * world)
            e.walks_init(starts, LT.DEEPWALK, 12, 7)
            comm = ltdist.TorchComm()
            ltdist.attach_peers(e, comm, len(starts))  # CUDA IPC between the processes
            if fused:  # speculative supersteps: the host reads the sent sum every 4th superstep
                counters = ltdist.run_supersteps_p2p_fused(e, comm, "cuda:0")
            else:
                counters = ltdist.run_supersteps_p2p(e, comm, "cpu")
            paths, lengths = e.partial_paths()
            paths, lengths = paths.cpu(), lengths.cpu()
            paths ^= ltdist.SIGN
            comm.allreduce_(paths, "min")
            paths ^= ltdist.SIGN
            comm.allreduce_(lengths, "max")
            if rank == 0:
                out_q.put((paths.numpy().view(np.uint32).copy(), lengths.numpy().view(np.uint32).copy(), counters))
    finally:
        tdist.destroy_process_group()


@pytest.mark.parametrize("fused", [False, True])
def test_peer_exchange_processes_cuda_ipc(gpu, fused):
    """Two processes on one GPU, each rank's receive buffers opened by the other through CUDA IPC
    (lt_ipc_handle / lt_ipc_open): the multi-process wiring of the peer exchange."""
    import socket

    import torch.multiprocessing as mp
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_p2p_proc, args=(r, 2, port, q, fused)) for r in range(2)]
    for p in procs:
        p.start()
    paths, lengths, counters = q.get(timeout=300)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    g = lt_inputs.rmat_cpu(13, 8 * 2 ** 13, seed=3)
    starts = lt_inputs.deepwalk_starts(2 * g.n, g.n)
    op, ol, _, _ = oracle_of(g, starts, LT.DEEPWALK, 12, 7)
    np.testing.assert_array_equal(lengths, ol)
    np.testing.assert_array_equal(paths, op)
    assert counters["records_sent"] > 0


@pytest.mark.parametrize("world", [2, 3, 4])
@pytest.mark.parametrize("layout", [LT.LAYOUT_CSR, LT.LAYOUT_ADJ])
@pytest.mark.parametrize("app,param", [(LT.DEEPWALK, 16), (LT.PPR, 0.15)])
def test_fused_superstep_exact(gpu, g13, world, layout, app, param):
    """lt_superstep_p2p (one owned partition per rank, one host round trip per superstep): merged
    paths equal the oracle, the same walks cross ranks as with the unfused loop, and a second epoch on
    the same engines works (parities stay aligned)."""
    import torch
    starts = (lt_inputs.deepwalk_starts(3 * g13.n, g13.n) if app == LT.DEEPWALK
              else lt_inputs.ppr_starts(20_000, g13.argmax_deg))
    hub = ltdist.ThreadComm.Hub(world)
    out, errors = [None] * world, []

    def rank_main(r):
        try:
            with LT.Engine(rank=r, world=world, layout=layout, chunk_walks=512, timing=True) as e:
                e.graph_load(g13.row_ptr, g13.col, world)
                comm = ltdist.ThreadComm(hub, r)
                res = []
                for seed in (2, 3):
                    e.walks_init(starts, app, param, seed)
                    if seed == 2:
                        ltdist.attach_peers(e, comm, len(starts))
                    cnt = ltdist.run_supersteps_p2p_fused(e, comm, "cuda")
                    paths, lengths = ltdist.merge_paths(e, comm)
                    torch.cuda.synchronize()
                    res.append((paths.cpu().numpy().view(np.uint32), lengths.cpu().numpy().view(np.uint32), cnt,
                                e.stats()))
                out[r] = res
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
    for i, seed in enumerate((2, 3)):
        op, ol, osteps, _ = oracle_of(g13, starts, app, param, seed)
        for r in range(world):
            paths, lengths, cnt, st = out[r][i]
            np.testing.assert_array_equal(lengths, ol)
            np.testing.assert_array_equal(paths, op)
        assert sum(out[r][i][3]["steps"] for r in range(world)) == osteps
        assert sum(out[r][i][2]["records_sent"] for r in range(world)) > 0
        # per-epoch statistics accumulate over the supersteps (one update launch each; the final
        # lt_run over the empty buckets launches none), so bytes / update_ms is the epoch's rate
        for r in range(world):
            st, cnt = out[r][i][3], out[r][i][2]
            assert st["update_launches"] == cnt["supersteps"]
            assert st["update_ms"] > 0 and st["run_ms"] > 0


def test_fused_superstep_preconditions(gpu, g13):
    with LT.Engine(rank=0, world=2) as e:
        e.graph_load(g13.row_ptr, g13.col, 4)  # two owned partitions
        e.walks_init(lt_inputs.deepwalk_starts(100, g13.n), LT.DEEPWALK, 5, 1)
        import torch
        sent = torch.zeros(1, dtype=torch.int64, device="cuda")
        with pytest.raises(LT.LTError):
            e.superstep_p2p(sent)  # not attached
        e.exchange_buffers(100)
        with pytest.raises(LT.LTError):
            e.superstep_p2p(sent)


def test_fused_superstep_overflow_is_an_error(gpu, g13):
    """A receive buffer too small for one superstep's arrivals: the fused loop still ends (the
    receiver inserts only what was stored) and the sending rank's final lt_run reports the overflow."""
    import torch
    world = 2
    hub = ltdist.ThreadComm.Hub(world)
    errors = []

    def rank_main(r):
        try:
            with LT.Engine(rank=r, world=world) as e:
                e.graph_load(g13.row_ptr, g13.col, world)
                e.walks_init(lt_inputs.deepwalk_starts(g13.n, g13.n), LT.DEEPWALK, 10, 1)
                comm = ltdist.ThreadComm(hub, r)
                ltdist.attach_peers(e, comm, 16)
                try:
                    ltdist.run_supersteps_p2p_fused(e, comm, "cuda")
                finally:
                    torch.cuda.synchronize()
        except LT.LTError as ex:
            errors.append(ex)

    th = [threading.Thread(target=rank_main, args=(r,)) for r in range(world)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    assert errors and all("overflow" in str(x) for x in errors)


@pytest.mark.parametrize("p2p", [False, True])
def test_ownership_paths_off_visit_counts(gpu, g13, p2p):
    """path_mode 2 (no path matrix, the paper's accounting) with range ownership: no path rows are
    pre-filled or merged, the visit counts summed over ranks equal the oracle's (the
    0xFF pre-fill once ran over the 8-entry placeholder)."""
    import torch
    world = 2
    starts = lt_inputs.deepwalk_starts(2 * g13.n, g13.n)
    hub = ltdist.ThreadComm.Hub(world)
    out, errors = [None] * world, []

    def rank_main(r):
        try:
            with LT.Engine(rank=r, world=world, path_mode=2, visit_counts=True, chunk_walks=512, timing=True) as e:
                e.graph_load(g13.row_ptr, g13.col, 8)
                e.walks_init_pagerank(starts, 12, 0.15, 9)
                comm = ltdist.ThreadComm(hub, r)
                if p2p:
                    ltdist.attach_peers(e, comm, len(starts))
                    cnt = ltdist.run_supersteps_p2p(e, comm, "cuda")
                else:
                    cnt = ltdist.run_supersteps(e, comm, "cuda")
                counts = ltdist.merge_visit_counts(e, comm, "cuda")
                torch.cuda.synchronize()
                assert e.pool_state()["device_err"] == 0
                out[r] = (counts.cpu().numpy().view(np.uint64), cnt, e.stats())
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
    op, ol, osteps, _ = O.walks(g13.row_ptr, g13.col, starts, app=O.PAGERANK, length=12, alpha=0.15, seed=9)
    expect = O.visit_counts(op, ol, g13.n)
    for counts, cnt, st in out:
        np.testing.assert_array_equal(counts, expect)
    assert sum(st["steps"] for _, _, st in out) == osteps
    assert all(st["update_launches"] >= 1 and st["update_ms"] > 0 for _, _, st in out)


@pytest.mark.parametrize("exchange", ["alltoall", "p2p", "fused"])
@pytest.mark.parametrize("layout", [LT.LAYOUT_CSR, LT.LAYOUT_ADJ])
def test_ownership_lane_refill_offset_records(gpu, g13, exchange, layout):
    """Range ownership on the lane-refill kernel at P > 1 (refill 2): walks for a local bucket leave as O
    records, walks for other ranks as V records (a receiver needs the vertex), through send buckets or
    straight into peer buffers."""
    world = 3
    starts = lt_inputs.deepwalk_starts(3 * g13.n, g13.n)
    P = world if exchange == "fused" else 12
    kw = dict(layout=layout, refill=2, chunk_walks=512)
    if exchange == "alltoall":
        res = run_owned(g13, starts, LT.DEEPWALK, 16, 2, P, world, **kw)
    else:
        res = run_owned_p2p(g13, starts, LT.DEEPWALK, 16, 2, P, world, **kw) if exchange == "p2p" else None
    if exchange == "fused":
        import torch
        hub = ltdist.ThreadComm.Hub(world)
        res, errors = [None] * world, []

        def rank_main(r):
            try:
                with LT.Engine(rank=r, world=world, **kw) as e:
                    e.graph_load(g13.row_ptr, g13.col, P)
                    e.walks_init(starts, LT.DEEPWALK, 16, 2)
                    comm = ltdist.ThreadComm(hub, r)
                    ltdist.attach_peers(e, comm, len(starts))
                    cnt = ltdist.run_supersteps_p2p_fused(e, comm, "cuda")
                    paths, lengths = ltdist.merge_paths(e, comm)
                    torch.cuda.synchronize()
                    res[r] = (paths.cpu().numpy().view(np.uint32), lengths.cpu().numpy().view(np.uint32), cnt,
                              e.stats())
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
    op, ol, osteps, _ = oracle_of(g13, starts, LT.DEEPWALK, 16, 2)
    for paths, lengths, _, _ in res:
        np.testing.assert_array_equal(lengths, ol)
        np.testing.assert_array_equal(paths, op)
    assert sum(r[3]["steps"] for r in res) == osteps


# ---- paths on the home rank (lt_paths_buffers / lt_paths_attach): every rank writes its path entries and
# lengths straight into rank 0's matrix, so the paths are complete there without a merge

@pytest.mark.parametrize("exchange", ["alltoall", "p2p", "fused"])
@pytest.mark.parametrize("app,param", [(LT.DEEPWALK, 16), (LT.PPR, 0.15)])
def test_paths_on_home_rank(gpu, g13, exchange, app, param):
    import torch
    world = 3
    starts = (lt_inputs.deepwalk_starts(3 * g13.n, g13.n) if app == LT.DEEPWALK
              else lt_inputs.ppr_starts(20_000, g13.argmax_deg))
    P = world if exchange == "fused" else 12
    hub = ltdist.ThreadComm.Hub(world)
    out, errors = [None] * world, []

    def rank_main(r):
        try:
            with LT.Engine(rank=r, world=world, layout=LT.LAYOUT_ADJ, chunk_walks=512, refill=2) as e:
                e.graph_load(g13.row_ptr, g13.col, P)
                comm = ltdist.ThreadComm(hub, r)
                res = []
                for seed in (2, 3):  # two epochs: the second reuses the attachment
                    e.walks_init(starts, app, param, seed)
                    ltdist.attach_paths(e, comm)
                    if exchange == "alltoall":
                        ltdist.run_supersteps(e, comm, "cuda")
                    else:
                        if seed == 2:
                            ltdist.attach_peers(e, comm, len(starts))
                        run = ltdist.run_supersteps_p2p_fused if exchange == "fused" else ltdist.run_supersteps_p2p
                        run(e, comm, "cuda")
                    torch.cuda.synchronize()
                    comm.allgather_obj(None)  # every rank's kernels are done
                    if r == 0:
                        paths, lengths = e.home_paths()
                        res.append((paths.cpu().numpy().view(np.uint32), lengths.cpu().numpy().view(np.uint32)))
                    else:
                        with pytest.raises(LT.LTError):
                            e.get_paths()  # the paths live on the home rank
                    assert e.stats()["steps"] >= 0
                out[r] = res
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
    for i, seed in enumerate((2, 3)):
        op, ol, _, _ = oracle_of(g13, starts, app, param, seed)
        paths, lengths = out[0][i]
        np.testing.assert_array_equal(lengths, ol)
        np.testing.assert_array_equal(paths, op)


def _home_proc(rank, world, port, out_q):
    import os

    import torch
    import torch.distributed as tdist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    tdist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        g = lt_inputs.rmat_cpu(13, 8 * 2 ** 13, seed=3)
        starts = lt_inputs.deepwalk_starts(2 * g.n, g.n)
        with LT.Engine(rank=rank, world=world) as e:
            e.graph_load(g.row_ptr, g.col, world)
            e.walks_init(starts, LT.DEEPWALK, 12, 7)
            comm = ltdist.TorchComm()
            ltdist.attach_paths(e, comm)  # CUDA IPC of rank 0's path matrix and length array
            ltdist.attach_peers(e, comm, len(starts))
            ltdist.run_supersteps_p2p_fused(e, comm, "cuda:0")
            torch.cuda.synchronize()
            tdist.barrier()
            if rank == 0:
                paths, lengths = e.home_paths()
                out_q.put((paths.cpu().numpy().view(np.uint32).copy(), lengths.cpu().numpy().view(np.uint32).copy()))
    finally:
        tdist.destroy_process_group()


def test_paths_on_home_rank_processes_cuda_ipc(gpu):
    import socket

    import torch.multiprocessing as mp
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_home_proc, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    paths, lengths = q.get(timeout=300)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    g = lt_inputs.rmat_cpu(13, 8 * 2 ** 13, seed=3)
    starts = lt_inputs.deepwalk_starts(2 * g.n, g.n)
    op, ol, _, _ = oracle_of(g, starts, LT.DEEPWALK, 12, 7)
    np.testing.assert_array_equal(lengths, ol)
    np.testing.assert_array_equal(paths, op)
