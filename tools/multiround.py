#!/usr/bin/env python3
"""SURVEY.md §8(f) f3 / PAPER.md:353-363 (Fig. 16): massive walk counts under a walk-pool cap. Three arms
with the same device memory cap m_w on the walk pool:
  * spill (lt_config.walk_spill, the paper's mechanism): every walk exists
    from the start; full chunks of the buckets with the fewest walks are evicted to pinned host memory
    and loaded back before their partition is computed;
  * admission (lt_config.walk_pool_walks alone): walks are created in index order as walks end;
  * multi-round baseline: the same walks in R sequential rounds of m_w (separate lt_walks_init + lt_run).

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
    ap.add_argument("--arms", default="spill,admission,multi")
    a = ap.parse_args()
    import torch
    import paper_conf_icde_xing0wxl23_b200 as LT
    c = lt_inputs.CONFIGS[a.config]
    torch.cuda.set_device(0)
    g = lt_inputs.rmat_gpu(c["scale"], c["tuples"], seed=1, permute=c["permute"])
    W = a.walks
    starts = torch.from_numpy(lt_inputs.deepwalk_starts(W, g.n).view(np.int32)).cuda()
    ooc = a.graph_pool_gb > 0

    arms = a.arms.split(",")

    def engine(cap, spill=False):
        return LT.Engine(path_mode=2, walk_pool_walks=cap, graph_pool_bytes=int(a.graph_pool_gb * 2 ** 30),
                         zero_copy=ooc, continue_resident=ooc, timing=True, walk_spill=spill)

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
        line = {"what": "walk spill vs walk admission vs multi-round (PAPER.md:353-363, Fig. 16 shape)",
                "graph": f"{c['name']} out-of-core P={a.partitions} pool={a.graph_pool_gb} GiB" if ooc
                else f"{c['name']} HBM-resident P={a.partitions}",
                "walks": W, "cap_walks": cap, "rounds": rounds, "length": a.length}

        def capped(spill):
            with engine(cap, spill) as e:
                e.graph_load(g.row_ptr, g.col, a.partitions)

                def go():
                    e.walks_init(starts, LT.DEEPWALK, a.length, 1)
                    e.run()
                    return e.stats()
                go()  # warm-up
                ms, st = min((timed(go) for _ in range(a.reps)), key=lambda x: x[0])
            assert st["steps"] == W * a.length
            out = {"ms": ms, "steps_per_s": st["steps"] / (ms / 1000), "admissions": st["admissions"],
                   "peak_live": st["peak_live"], "graph_h2d_gb": st["graph_h2d_bytes"] / 1e9,
                   "explicit_copies": st["explicit_copies"], "iterations": st["iterations"],
                   "chunks_total": st["chunks_total"], "update_launches": st["update_launches"]}
            out.update(update_ms=st["update_ms"], run_ms=st["run_ms"], load_ms=st["load_ms"],
                       host_syncs=st["host_syncs"])
            if spill:
                out.update(spilled_chunks=st["spilled_chunks"], reloaded_chunks=st["reloaded_chunks"],
                           spill_d2h_gb=st["spill_d2h_bytes"] / 1e9, spill_h2d_gb=st["spill_h2d_bytes"] / 1e9,
                           host_chunks_peak=st["host_chunks_peak"], spill_xfer_ms=st["spill_xfer_ms"],
                           spill_prefetched_chunks=st["spill_prefetched_chunks"])
            return out

        # (1) walk spill (every walk exists; the pool evicts to host memory) and (2) walk admission
        if "spill" in arms:
            line["spill"] = capped(True)
        if "admission" in arms:
            line["admission"] = capped(False)
        if "multi" not in arms:
            print(json.dumps(line), flush=True)
            continue
        # (3) multi-round baseline: R rounds of `cap` walks (walk IDs continue across rounds)
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
        line["multi_round"] = {"ms": ms_mr, "steps_per_s": mt["steps"] / (ms_mr / 1000),
                               "graph_h2d_gb": mt["graph_h2d_bytes"] / 1e9, "explicit_copies": mt["explicit_copies"],
                               "iterations": mt["iterations"]}
        for arm in ("spill", "admission"):
            if arm in line:
                line[f"multi_round_slowdown_vs_{arm}"] = ms_mr / line[arm]["ms"]
        assert mt["steps"] == W * a.length
        print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
