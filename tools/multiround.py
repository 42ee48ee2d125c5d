#!/usr/bin/env python3
"""SURVEY.md §8(f) f3 / PAPER.md:353-363 (Fig. 16): massive walk counts under a walk-pool cap, walk
admission (lt_config.walk_pool_walks) against the multi-round baseline (the same walks in R sequential
rounds of W/R, each a separate lt_walks_init + lt_run) with the same memory cap.

Graph: BASELINE configs[3] (FS-shaped R-MAT s26), out of core (pinned host CSR, capped graph pool,
adaptive zero copy, continuation into resident partitions). Walks: DeepWalk l = 10 (the paper's Fig. 15
setting), starts w mod n, no path matrix (path_mode 2, the paper's accounting, :287). Device-timed with
CUDA events; one JSON line per case."""
import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import lt_inputs  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=4)
    ap.add_argument("--walks", type=int, default=800_000_000)
    ap.add_argument("--caps", default="100000000,200000000,400000000")
    ap.add_argument("--length", type=int, default=10)
    ap.add_argument("--partitions", type=int, default=64)
    ap.add_argument("--graph-pool-gb", type=float, default=8.0)
    ap.add_argument("--reps", type=int, default=1)
    a = ap.parse_args()
    import torch
    import paper_conf_icde_xing0wxl23_b200 as LT
    c = lt_inputs.CONFIGS[a.config]
    torch.cuda.set_device(0)
    g = lt_inputs.rmat_gpu(c["scale"], c["tuples"], seed=1, permute=c["permute"])
    W = a.walks
    starts = torch.from_numpy(lt_inputs.deepwalk_starts(W, g.n).view(np.int32)).cuda()
    ooc = a.graph_pool_gb > 0

    def engine(cap):
        return LT.Engine(path_mode=2, walk_pool_walks=cap, graph_pool_bytes=int(a.graph_pool_gb * 2 ** 30),
                         zero_copy=True, continue_resident=True, timing=True)

    def timed(fn):
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        out = fn()
        e1.record()
        torch.cuda.synchronize()
        return e0.elapsed_time(e1), out

    for cap in [int(x) for x in a.caps.split(",")]:
        rounds = -(-W // cap)
        # (1) walk admission: all W walks, at most `cap` live
        with engine(cap) as e:
            t0 = time.time()
            e.graph_load(g.row_ptr, g.col, a.partitions)
            load_s = time.time() - t0

            def adm():
                e.walks_init(starts, LT.DEEPWALK, a.length, 1)
                e.run()
                return e.stats()
            adm()  # warm-up
            ms_adm, st = min((timed(adm) for _ in range(a.reps)), key=lambda x: x[0])
        # (2) multi-round baseline: R rounds of `cap` walks (walk IDs continue across rounds)
        with engine(0) as e:
            e.graph_load(g.row_ptr, g.col, a.partitions)

            def multi():
                tot = {"steps": 0, "graph_h2d_bytes": 0, "explicit_copies": 0, "iterations": 0}
                for r in range(rounds):
                    lo, hi = r * cap, min(W, (r + 1) * cap)
                    e.walks_init(starts[lo:hi], LT.DEEPWALK, a.length, 1, lo)
                    e.run()
                    s = e.stats()
                    for k in tot:
                        tot[k] += s[k]
                return tot
            multi()
            ms_mr, mt = min((timed(multi) for _ in range(a.reps)), key=lambda x: x[0])
        line = {"what": "walk admission vs multi-round (PAPER.md:353-363, Fig. 16 shape)",
                "graph": f"{c['name']} out-of-core P={a.partitions} pool={a.graph_pool_gb} GiB" if ooc else c["name"],
                "walks": W, "cap_walks": cap, "rounds": rounds, "length": a.length,
                "admission": {"ms": ms_adm, "steps_per_s": st["steps"] / (ms_adm / 1000),
                              "admissions": st["admissions"], "peak_live": st["peak_live"],
                              "graph_h2d_gb": st["graph_h2d_bytes"] / 1e9, "explicit_copies": st["explicit_copies"],
                              "iterations": st["iterations"], "chunks_total": st["chunks_total"]},
                "multi_round": {"ms": ms_mr, "steps_per_s": mt["steps"] / (ms_mr / 1000),
                                "graph_h2d_gb": mt["graph_h2d_bytes"] / 1e9, "explicit_copies": mt["explicit_copies"],
                                "iterations": mt["iterations"]},
                "multi_round_slowdown": ms_mr / ms_adm, "graph_load_s": round(load_s, 1)}
        assert st["steps"] == mt["steps"] == W * a.length
        print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
