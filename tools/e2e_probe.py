#!/usr/bin/env python3
"""Wall-clock probe of the end-to-end copy-out paths (lt_run_to_host / lt_run_to_host_compact) on one
BASELINE config: per call time, stats, and the phase split. Diagnostics only, not bench values."""
import argparse
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import lt_inputs  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=3)
    ap.add_argument("--chunks", default="1,4,16")
    a = ap.parse_args()
    import torch
    import paper_conf_icde_xing0wxl23_b200 as LT
    c = lt_inputs.CONFIGS[a.config]
    g = lt_inputs.rmat_gpu(c["scale"], c["tuples"], seed=1, permute=c["permute"])
    W = g.n
    if c["app"] == "ppr":
        st, app, prm, S = lt_inputs.ppr_starts(W, g.argmax_deg), LT.PPR, c["alpha"], 128
    else:
        st, app, prm, S = lt_inputs.deepwalk_starts(W, g.n), LT.DEEPWALK, c["length"], c["length"] + 1
    hs = torch.from_numpy(st.view(np.int32)).pin_memory()
    t0 = time.time()
    ho = torch.empty(W + 1, dtype=torch.int64, pin_memory=True)
    hv = torch.empty(W * S, dtype=torch.int32, pin_memory=True)
    print(f"pinned alloc {time.time() - t0:.2f} s", flush=True)
    with LT.Engine() as e:
        e.graph_load(g.row_ptr, g.col, 1)
        for ch in [int(x) for x in a.chunks.split(",")]:
            for rep in range(2):
                torch.cuda.synchronize()
                t0 = time.time()
                e.run_to_host_compact(hs, app, prm, 1, 0, offsets=ho, vertices=hv, chunks=ch)
                dt = time.time() - t0
                s = e.stats()
                print(f"compact chunks={ch} rep={rep}: {dt * 1000:.1f} ms, steps {s['steps']}, run_ms {s['run_ms']:.1f}, "
                      f"init_ms {s['init_ms']:.1f}, d2h {s['d2h_bytes'] / 1e9:.2f} GB", flush=True)
        e.walks_init(hs, app, prm, 1)
        torch.cuda.synchronize()
        t0 = time.time()
        e.walks_init(hs, app, prm, 1)
        e.run()
        torch.cuda.synchronize()
        t1 = time.time()
        o, v = e.get_paths_compact()
        t2 = time.time()
        print(f"init+run {1000 * (t1 - t0):.1f} ms; get_paths_compact (pageable numpy) {1000 * (t2 - t1):.1f} ms")


if __name__ == "__main__":
    main()
