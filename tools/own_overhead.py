#!/usr/bin/env python3
"""Range-ownership superstep overhead on ONE GPU: `world` engines in threads (dist.ThreadComm), all on
cuda:0, DeepWalk l=80 over |V| walks of a BASELINE config's graph. Prints one JSON line: wall time of
the superstep loop, supersteps, and the host-side share (wall minus the summed update-kernel time).
--p2p runs the peer exchange (walks appended into the owner's receive buffer by the update kernels).
--legacy runs the superstep loop of the first version (all-to-all of counts, then an all-reduce for
termination); pair it with LT_LIBRARY pointing at a build of that version (synchronising pack /
insert / pending). Not a multi-GPU number: the ranks share one device."""
import argparse
import json
import os
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import lt_inputs  # noqa: E402


def legacy_supersteps(engine, comm, device):
    from paper_conf_icde_xing0wxl23_b200 import dist as ltdist
    cache, supersteps = {}, 0
    while True:
        engine.run()
        buf = ltdist.send_buffer(engine, device, cache)
        counts = engine.exchange_pack(buf)
        recv_counts = comm.alltoall_counts(counts, device)
        recv = comm.alltoallv(buf, counts, recv_counts)
        engine.exchange_insert(recv, sum(recv_counts))
        crossed = comm.allreduce_sum(sum(recv_counts), device)
        supersteps += 1
        if crossed == 0:
            return {"supersteps": supersteps}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=2)
    ap.add_argument("--world", type=int, default=2)
    ap.add_argument("--partitions", type=int, default=0, help="0: one per rank")
    ap.add_argument("--legacy", action="store_true")
    ap.add_argument("--p2p", action="store_true", help="peer exchange (dist.run_supersteps_p2p)")
    ap.add_argument("--fused", action="store_true", help="peer exchange, fused superstep (run_supersteps_p2p_fused)")
    ap.add_argument("--reps", type=int, default=2)
    ap.add_argument("--refill", type=int, default=0, help="lt_config.refill: 0 auto, 1 off, 2 on")
    a = ap.parse_args()
    import torch

    import paper_conf_icde_xing0wxl23_b200 as LT
    from paper_conf_icde_xing0wxl23_b200 import dist as ltdist
    c = lt_inputs.CONFIGS[a.config]
    g = lt_inputs.rmat_gpu(c["scale"], c["tuples"], seed=1, permute=c["permute"], device=0)
    starts = torch.from_numpy(lt_inputs.deepwalk_starts(g.n, g.n).view(np.int32)).cuda()
    P = a.partitions or a.world
    out = {}

    def rank_main(r, hub, res):
        with LT.Engine(rank=r, world=a.world, timing=True, refill=a.refill) as e:
            e.graph_load(g.row_ptr, g.col, P)
            comm = ltdist.ThreadComm(hub, r)
            if a.p2p or a.fused:
                e.walks_init(starts, LT.DEEPWALK, 80, 1)
                ltdist.attach_peers(e, comm, g.n)
            for rep in range(a.reps + 1):
                e.walks_init(starts, LT.DEEPWALK, 80, 1)
                hub.barrier.wait()
                torch.cuda.synchronize()
                t0 = time.perf_counter()
                upd = 0.0
                if a.legacy:
                    cnt = legacy_supersteps(e, comm, "cuda")
                elif a.fused:
                    cnt = ltdist.run_supersteps_p2p_fused(e, comm, "cuda")
                elif a.p2p:
                    cnt = ltdist.run_supersteps_p2p(e, comm, "cuda")
                else:
                    cnt = ltdist.run_supersteps(e, comm, "cuda")
                torch.cuda.synchronize()
                hub.barrier.wait()
                if rep:  # rep 0 is warm-up
                    res[r].append((time.perf_counter() - t0, cnt["supersteps"], e.stats()["steps"]))

    hub = ltdist.ThreadComm.Hub(a.world)
    res = [[] for _ in range(a.world)]
    th = [threading.Thread(target=rank_main, args=(r, hub, res)) for r in range(a.world)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    wall = min(max(res[r][i][0] for r in range(a.world)) for i in range(a.reps))
    ss = res[0][-1][1]
    out = {"config": a.config, "world": a.world, "partitions": P, "legacy": a.legacy, "p2p": a.p2p, "fused": a.fused, "refill": a.refill,
           "wall_ms": wall * 1e3,
           "supersteps": ss, "ms_per_superstep": wall * 1e3 / ss, "n": g.n,
           "library": os.environ.get("LT_LIBRARY", "liblt.so")}
    print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
