"""Range-ownership protocol over real torch.distributed collectives on CPU (gloo, world size 2 and 3):
dist.run_supersteps + TorchComm + dist.merge_paths, each rank driving a CPU stand-in engine
(tests/cpu_owner_engine.py). The merged paths must equal the oracle's bit-exactly, whatever the
number of ranks: the counter-based RNG makes a walk independent of where it runs."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

import lt_inputs
import oracle as O
import paper_conf_icde_xing0wxl23_b200 as LT


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, app, param, P, out_q):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
    import torch.distributed as dist

    from cpu_owner_engine import CpuOwnerEngine
    from paper_conf_icde_xing0wxl23_b200 import dist as ltdist

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        g = lt_inputs.rmat_cpu(9, 3000, seed=5)
        W = 700
        starts = lt_inputs.ppr_starts(W, g.argmax_deg) if app == LT.PPR else lt_inputs.deepwalk_starts(W, g.n)
        eng = CpuOwnerEngine(g, P, rank, world)
        if app == LT.PAGERANK:
            eng.walks_init_pagerank(starts, 12, param, 11)
        else:
            eng.walks_init(starts, app, param, 11)
        comm = ltdist.TorchComm()
        counters = ltdist.run_supersteps(eng, comm, "cpu")
        paths, lengths = ltdist.merge_paths(eng, comm)
        counts = ltdist.merge_visit_counts(eng, comm, "cpu")
        if rank == 0:
            out_q.put((paths.numpy().view(np.uint32).copy(), lengths.numpy().view(np.uint32).copy(), counters,
                       counts.numpy().view(np.uint64).copy()))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
@pytest.mark.parametrize("app,param", [(LT.DEEPWALK, 12), (LT.PPR, 0.2), (LT.PAGERANK, 0.3)])
def test_ownership_protocol_gloo(world, app, param):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    P = 6
    procs = [ctx.Process(target=_worker, args=(r, world, port, app, param, P, q)) for r in range(world)]
    for p in procs:
        p.start()
    paths, lengths, counters, counts = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    g = lt_inputs.rmat_cpu(9, 3000, seed=5)
    W = 700
    starts = lt_inputs.ppr_starts(W, g.argmax_deg) if app == LT.PPR else lt_inputs.deepwalk_starts(W, g.n)
    kw = {LT.DEEPWALK: dict(app=O.DEEPWALK, length=12), LT.PPR: dict(app=O.PPR, alpha=0.2),
          LT.PAGERANK: dict(app=O.PAGERANK, length=12, alpha=0.3)}[app]
    op, ol, _, _ = O.walks(g.row_ptr, g.col, starts, seed=11, **kw)
    np.testing.assert_array_equal(lengths, ol)
    np.testing.assert_array_equal(paths, op)
    np.testing.assert_array_equal(counts, O.visit_counts(op, ol, g.n))  # summed over ranks
    assert counters["supersteps"] >= 2 and counters["records_sent"] > 0


def _worker_p2p(rank, world, port, app, param, P, out_q, fused=False):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
    import torch.distributed as dist

    from cpu_owner_engine import CpuOwnerEngine
    from paper_conf_icde_xing0wxl23_b200 import dist as ltdist

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    eng = None
    try:
        g = lt_inputs.rmat_cpu(9, 3000, seed=5)
        W = 700
        starts = lt_inputs.ppr_starts(W, g.argmax_deg) if app == LT.PPR else lt_inputs.deepwalk_starts(W, g.n)
        eng = CpuOwnerEngine(g, P, rank, world)
        comm = ltdist.TorchComm()
        res = []
        for seed in (11, 12):  # two epochs: the parities stay aligned
            eng.walks_init(starts, app, param, seed)
            if seed == 11:
                ltdist.attach_peers(eng, comm, W)
            if fused:  # one owned partition per rank; the host reads the sum every 4th superstep
                counters = ltdist.run_supersteps_p2p_fused(eng, comm, "cpu")
            else:
                counters = ltdist.run_supersteps_p2p(eng, comm, "cpu")
            paths, lengths = ltdist.merge_paths(eng, comm)
            res.append((paths.numpy().view(np.uint32).copy(), lengths.numpy().view(np.uint32).copy(), counters))
        dist.barrier()
        if rank == 0:
            out_q.put(res)
    finally:
        if eng is not None and hasattr(eng, "_own_shm"):
            dist.barrier()
            eng.close_exchange()
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
@pytest.mark.parametrize("app,param", [(LT.DEEPWALK, 12), (LT.PPR, 0.2)])
@pytest.mark.parametrize("fused", [False, True])
def test_peer_exchange_protocol_gloo(world, app, param, fused):
    """dist.attach_peers + run_supersteps_p2p over gloo (the CPU stand-in emulates the receive buffers
    with shared memory): merged paths equal the oracle over two epochs."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    P = world if fused else 8
    procs = [ctx.Process(target=_worker_p2p, args=(r, world, port, app, param, P, q, fused)) for r in range(world)]
    for p in procs:
        p.start()
    res = q.get(timeout=300)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    g = lt_inputs.rmat_cpu(9, 3000, seed=5)
    W = 700
    starts = lt_inputs.ppr_starts(W, g.argmax_deg) if app == LT.PPR else lt_inputs.deepwalk_starts(W, g.n)
    for (paths, lengths, counters), seed in zip(res, (11, 12)):
        kw = dict(app=O.DEEPWALK, length=param) if app == LT.DEEPWALK else dict(app=O.PPR, alpha=param)
        op, ol, _, _ = O.walks(g.row_ptr, g.col, starts, seed=seed, **kw)
        np.testing.assert_array_equal(lengths, ol)
        np.testing.assert_array_equal(paths, op)
        assert counters["records_sent"] > 0
