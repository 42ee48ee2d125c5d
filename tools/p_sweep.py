#!/usr/bin/env python3
"""Partition-count sweep of the update kernels on one GPU (DESIGN.md §8 "P > 1"): BASELINE configs[3]
(FS-shaped R-MAT s26, |V| DeepWalk walks of length 80; --config picks another), one JSON line per
(kernel, P): steps/s device-timed over --steps walks after --warmup, visits per step, sweeps, launches.
  refill 0 = batch kernel (k_update), 2 = lane refill (k_update_rf)."""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import lt_inputs  # noqa: E402
import paper_conf_icde_xing0wxl23_b200 as LT  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=4)
    ap.add_argument("--P", default="4,8,16,64")
    ap.add_argument("--refill", default="0,2")
    ap.add_argument("--layout", type=int, default=0)
    ap.add_argument("--app", default="config")
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=1)
    ap.add_argument("--chunk-walks", type=int, default=8192)
    ap.add_argument("--insert-mode", default="0")
    ap.add_argument("--parity", type=int, default=20000, help="sampled walks checked against the oracle (0: off)")
    ap.add_argument("--walks-mult", type=float, default=1.0, help="W = mult x |V| (launch-size sensitivity)")
    a = ap.parse_args()
    import torch
    c = lt_inputs.CONFIGS[a.config]
    g = lt_inputs.rmat_gpu(c["scale"], c["tuples"], seed=1, permute=c["permute"])
    app = c["app"] if a.app == "config" else a.app
    W = int(g.n * a.walks_mult)
    starts = (lt_inputs.deepwalk_starts(W, g.n) if app in ("deepwalk", "pagerank") else lt_inputs.ppr_starts(W, g.argmax_deg))
    sd = torch.from_numpy(starts.view(np.int32)).cuda()
    host = None
    for P in [int(x) for x in a.P.split(",")]:
        for rf in [int(x) for x in a.refill.split(",")]:
            for im in [int(x) for x in a.insert_mode.split(",")]:
                with LT.Engine(layout=a.layout, refill=rf, timing=True, chunk_walks=a.chunk_walks, insert_mode=im,
                               visit_counts=app == "pagerank") as e:
                    e.graph_load(g.row_ptr, g.col, P)

                    def one():
                        if app == "deepwalk":
                            e.walks_init(sd, LT.DEEPWALK, c.get("length", 80), 1)
                        elif app == "pagerank":
                            e.walks_init_pagerank(sd, c.get("length", 80), 0.15, 1)
                        else:
                            e.walks_init(sd, LT.PPR, c.get("alpha", 0.15), 1)
                        e.run()
                        return e.stats()

                    for _ in range(a.warmup):
                        one()
                    torch.cuda.synchronize()
                    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    ev0.record()
                    sts = [one() for _ in range(a.steps)]
                    ev1.record()
                    torch.cuda.synchronize()
                    ms = ev0.elapsed_time(ev1)
                    steps = sum(s["steps"] for s in sts)
                    line = {"config": a.config, "app": app, "P": P, "refill": rf, "insert_mode": im, "walks": W,
                            "kernel": {0: "k_update", 1: "k_update", 2: "k_update_rf"}[rf],
                            "layout": sts[-1]["layout"], "steps_per_s": steps / (ms / 1e3), "ms_per_step": ms / a.steps,
                            "update_ms_per_step": sum(s["update_ms"] for s in sts) / a.steps,
                            "visits_per_step": sum(s["visits"] for s in sts) / max(1, steps),
                            "sweeps": sts[-1]["sweeps"], "update_launches": sts[-1]["update_launches"]}
                    if a.parity:
                        import oracle as O
                        if host is None:
                            host = (g.row_ptr.cpu().numpy().view(np.uint64), g.col.cpu().numpy().view(np.uint32))
                        ids = np.unique(np.random.default_rng(P).integers(0, W, a.parity)).astype(np.uint64)
                        gp, gl = e.get_paths_rows(ids)
                        kw = dict(app={"deepwalk": O.DEEPWALK, "ppr": O.PPR, "pagerank": O.PAGERANK}[app],
                                  length=c.get("length", 80), alpha=c.get("alpha", 0.15), seed=1, ids=ids)
                        op, ol, _, _ = O.walks(host[0], host[1], starts[ids.astype(np.int64)], **kw)
                        line["parity_sample"] = {"walks": int(len(ids)),
                                                 "mismatched": int(np.sum(np.any(gp != op, axis=1) | (gl != ol)))}
                    print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
