#!/usr/bin/env python3
"""Minimal driver for ncu captures: generate one BASELINE.json config on the GPU, then run `--steps`
steps (lt_walks_init + lt_run) with nothing else on the device. Use with
  ncu --set full -k regex:k_update -s <warm launches> -c 1 python tools/profile_run.py ...
Numbers printed under a profiler are never bench values."""
import argparse
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import lt_inputs  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=4)
    ap.add_argument("--partitions", type=int, default=1)
    ap.add_argument("--steps", type=int, default=2)
    ap.add_argument("--chunk-walks", type=int, default=8192)
    ap.add_argument("--scale", type=int, default=None)
    ap.add_argument("--tuples", type=int, default=None)
    ap.add_argument("--l2-fetch", type=int, default=0)
    ap.add_argument("--gather-mode", type=int, default=3)
    ap.add_argument("--ilp", type=int, default=0)
    ap.add_argument("--blocks-per-sm", type=int, default=0)
    ap.add_argument("--layout", type=int, default=0)
    ap.add_argument("--path-mode", type=int, default=0)
    ap.add_argument("--refill", type=int, default=0)
    ap.add_argument("--app", default="config", choices=["config", "pagerank"])
    ap.add_argument("--restart-p", type=float, default=0.15)
    a = ap.parse_args()
    import torch

    import paper_conf_icde_xing0wxl23_b200 as LT
    c = dict(lt_inputs.CONFIGS[a.config])
    if a.scale:
        c["scale"] = a.scale
    if a.tuples:
        c["tuples"] = a.tuples
    torch.cuda.set_device(0)
    g = lt_inputs.rmat_gpu(c["scale"], c["tuples"], seed=1, permute=c["permute"])
    W = 4096 if c["walks"] == "4096" else g.n
    if c["app"] == "deepwalk":
        st, app, prm = lt_inputs.deepwalk_starts(W, g.n), LT.DEEPWALK, c["length"]
    else:
        st, app, prm = lt_inputs.ppr_starts(W, g.argmax_deg), LT.PPR, c["alpha"]
    sd = torch.from_numpy(st.view(np.int32)).cuda()
    with LT.Engine(chunk_walks=a.chunk_walks, l2_fetch_bytes=a.l2_fetch, timing=True,
                   gather_mode=a.gather_mode, ilp=a.ilp, blocks_per_sm=a.blocks_per_sm,
                   layout=a.layout, path_mode=a.path_mode,
                   refill=a.refill, visit_counts=a.app == "pagerank") as e:
        e.graph_load(g.row_ptr, g.col, a.partitions)
        for _ in range(a.steps):
            if a.app == "pagerank":  # random walk with restart + visit counts
                e.walks_init_pagerank(sd, int(c.get("length", 80)), a.restart_p, 1)
            else:
                e.walks_init(sd, app, prm, 1)
            e.run()
        s = e.stats()
    torch.cuda.synchronize()
    print({k: s[k] for k in ("steps", "visits", "sweeps", "update_launches", "run_ms", "update_ms", "layout",
                                 "graph_prep_ms")})


if __name__ == "__main__":
    main()
